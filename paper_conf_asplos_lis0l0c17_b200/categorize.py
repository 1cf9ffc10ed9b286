"""Inter-CTA locality categorizer and optimisation selector (paper section 4.4,
Figure 11: P:2265; bypassing P:2267; prefetching P:2271), B200 form.

The paper's framework estimates where a kernel's inter-CTA locality comes from
before choosing optimisations:

1. impose a new CTA order with Redirection-based clustering (Listing 4, X- and
   Y-partition) on a reduced problem and check whether performance and/or the
   L1 hit rate change -- "an indicator for inter-CTA locality potential";
   kernels with potential are algorithm- or cache-line-related;
2. turn L1 on/off: "if L2 cache access is significantly reduced after turning
   off L1 ... cache-line related";
3. no change in L2 transactions: high coalescing degree -> streaming, low ->
   data-related;
4. reads and writes of the same array with shifted references -> writing-related.

Exploitable kernels (algorithm, cache-line) then get CTA clustering in the
partition the probe favoured, throttling (TOT) and bypassing of the streaming
operand (BPS); the others get prefetching with the reshaped order (PFH) and
throttling (section 4.3).

`categorize` is the decision tree as a pure function of measured signals (the
paper gives no numeric thresholds; R21 states the ones used here).
The signals come either from ncu metric CSVs (`probe_from_ncu_csv`, as the
paper reads the CUDA profiler) or, lacking a profiler, from in-process timing
alone (`probe_timing`).  `tune` runs the optimisation set the verdict names,
sweeping the number of active agents over 1..max ("Opt Agents" in Table 2,
reading C11), and returns the fastest configuration.  No arithmetic of the
kernels happens here: everything runs through `ops` / the C ABI.
"""
from __future__ import annotations

import csv
import dataclasses
from dataclasses import dataclass, field
from typing import Callable

CATEGORIES = ("algorithm", "cache-line", "data", "writing", "streaming")   # section 3.2, Fig. 4


@dataclass
class Probe:
    """Measured signals of one kernel variant (any may be unknown)."""
    time_ms: float | None = None
    l1_hit_pct: float | None = None          # l1tex__t_sector_hit_rate.pct
    l2_sectors: float | None = None          # lts__t_sectors_srcunit_tex.sum
    ld_efficiency_pct: float | None = None   # smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct


@dataclass
class Signals:
    default: Probe                     # hardware CTA order
    rd_x: Probe                        # Redirection, X-partition (column-major; CC_ORDER_COL)
    rd_y: Probe                        # Redirection, Y-partition (row-major; CC_ORDER_ROW)
    l1_on: Probe | None = None         # streaming operand through L1
    l1_off: Probe | None = None        # streaming operand bypassing L1 (TMA / no_allocate)
    writes_shifted_reads: bool = False  # static reference analysis (step 4)


@dataclass
class Thresholds:
    """What counts as a "significant" change (the paper gives no numbers; R21)."""
    l1_hit_pp: float = 3.0            # L1 hit rate, percentage points
    l2_rel: float = 0.05              # L2 sectors, relative
    time_rel: float = 0.05            # time, relative
    coalesced_efficiency_pct: float = 50.0   # global-load efficiency at or above: "high" coalescing


@dataclass
class Verdict:
    category: str
    partition: str | None              # "col" (X-P) / "row" (Y-P) for exploitable kernels
    potential: bool
    optimizations: list[str]
    reasons: list[str] = field(default_factory=list)

    def as_dict(self):
        return dataclasses.asdict(self)


def _rel(a, b):
    return abs(a - b) / b if (a is not None and b is not None and b) else None


def categorize(sig: Signals, th: Thresholds | None = None) -> Verdict:
    """Figure 11's estimation step, in the text's order."""
    th = th or Thresholds()
    d = sig.default
    reasons: list[str] = []
    potential = False
    # step 1: does an imposed order (RD X / RD Y) change performance or L1 hit rate?
    for name, rd in (("RD-X", sig.rd_x), ("RD-Y", sig.rd_y)):
        if rd.l1_hit_pct is not None and d.l1_hit_pct is not None and \
                abs(rd.l1_hit_pct - d.l1_hit_pct) >= th.l1_hit_pp:
            potential = True
            reasons.append(f"{name} moves L1 hit rate {d.l1_hit_pct:.1f}% -> {rd.l1_hit_pct:.1f}%")
        r = _rel(rd.l2_sectors, d.l2_sectors)
        if r is not None and r >= th.l2_rel:
            potential = True
            reasons.append(f"{name} changes L2 sectors by {100 * (rd.l2_sectors / d.l2_sectors - 1):+.1f}%")
        r = _rel(rd.time_ms, d.time_ms)
        if r is not None and r >= th.time_rel:
            potential = True
            reasons.append(f"{name} changes time by {100 * (rd.time_ms / d.time_ms - 1):+.1f}%")
    if potential:
        # partition: the RD order with significantly fewer L2 sectors (the
        # better indicator), else the faster one, else Y (row)
        x, y = sig.rd_x, sig.rd_y
        r = _rel(x.l2_sectors, y.l2_sectors)
        if r is not None and r >= th.l2_rel:
            part = "col" if x.l2_sectors < y.l2_sectors else "row"
        elif x.time_ms is not None and y.time_ms is not None and x.time_ms != y.time_ms:
            part = "col" if x.time_ms < y.time_ms else "row"
        else:
            part = "row"
        # step 2: L1 off significantly reduces L2 accesses -> cache-line related
        cat = "algorithm"
        if sig.l1_on is not None and sig.l1_off is not None:
            r = _rel(sig.l1_off.l2_sectors, sig.l1_on.l2_sectors)
            if r is not None and sig.l1_off.l2_sectors < sig.l1_on.l2_sectors and r >= th.l2_rel:
                cat = "cache-line"
                reasons.append(f"L1 off cuts L2 sectors by {100 * r:.1f}%")
            else:
                reasons.append("L1 on/off leaves L2 sectors unchanged (sector-granular L1 fills)")
        return Verdict(cat, part, True, ["CLU", "TOT", "BPS"], reasons)
    reasons.append("no imposed order changes performance, L1 hit rate or L2 sectors")
    # step 4 (static): shifted self-references -> writing related
    if sig.writes_shifted_reads:
        return Verdict("writing", None, False, ["PFH", "TOT"], reasons + ["reads and writes one array, shifted"])
    # step 3: coalescing degree separates streaming from data related
    eff = d.ld_efficiency_pct
    if eff is None:
        reasons.append("coalescing degree unknown: taken as streaming")
        return Verdict("streaming", None, False, ["PFH", "TOT"], reasons)
    if eff >= th.coalesced_efficiency_pct:
        reasons.append(f"global-load efficiency {eff:.0f}% (coalesced)")
        return Verdict("streaming", None, False, ["PFH", "TOT"], reasons)
    reasons.append(f"global-load efficiency {eff:.0f}% (scattered)")
    return Verdict("data", None, False, ["PFH", "TOT"], reasons)


# ---------------------------------------------------------------- signal sources
NCU_METRICS = ("gpu__time_duration.sum", "l1tex__t_sector_hit_rate.pct", "lts__t_sectors_srcunit_tex.sum",
               "smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct")


def probe_from_ncu_csv(path: str) -> Probe:
    """A Probe from `ncu --csv --metrics <NCU_METRICS>` output; metrics summed
    (time, sectors) or launch-weighted (rates) over every captured launch."""
    rows = list(csv.reader(open(path)))
    hdr = [r for r in rows if r and r[0] == "ID"]
    if not hdr:
        raise ValueError(f"{path}: no ncu metric rows")
    h = hdr[0]
    per: dict[str, dict[str, float]] = {}
    for r in rows:
        if len(r) != len(h) or r[0] == "ID":
            continue
        d = dict(zip(h, r))
        try:
            v = float(d["Metric Value"].replace(",", ""))
        except ValueError:
            continue
        unit = d.get("Metric Unit", "")
        if d["Metric Name"] == "gpu__time_duration.sum":
            v *= {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3}.get(unit, 1e-6)
        per.setdefault(d["ID"], {})[d["Metric Name"]] = v
    launches = list(per.values())

    def tot(m):
        vals = [x[m] for x in launches if m in x]
        return sum(vals) if vals else None

    def wmean(m):                      # weight rates by launch time
        vals = [(x[m], x.get("gpu__time_duration.sum", 1.0)) for x in launches if m in x]
        w = sum(t for _, t in vals)
        return sum(v * t for v, t in vals) / w if vals and w else None

    return Probe(time_ms=tot("gpu__time_duration.sum"), l1_hit_pct=wmean("l1tex__t_sector_hit_rate.pct"),
                 l2_sectors=tot("lts__t_sectors_srcunit_tex.sum"),
                 ld_efficiency_pct=wmean("smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct"))


def time_ms(fn: Callable[[], object], reps: int = 10, warm: int = 3) -> float:
    """Median device time of fn() by CUDA events on the current stream."""
    import torch
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    out = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        out.append(a.elapsed_time(b))
    out.sort()
    return out[len(out) // 2]


def probe_timing(run: Callable[..., object], reps: int = 10, has_l1_staging: bool = True,
                 writes_shifted_reads: bool = False) -> Signals:
    """Signals from timing only: run(**launch kwargs) launches the kernel."""
    t = lambda **kw: Probe(time_ms=time_ms(lambda: run(**kw), reps))
    return Signals(default=t(backend="default"), rd_x=t(backend="redirect", order="col"),
                   rd_y=t(backend="redirect", order="row"),
                   l1_on=t(backend="default", staging="l1") if has_l1_staging else None,
                   l1_off=t(backend="default", staging="tma") if has_l1_staging else None,
                   writes_shifted_reads=writes_shifted_reads)


# ---------------------------------------------------------------- optimisation
def candidates(v: Verdict, max_agents: int, has_staging: bool = True) -> list[tuple[str, dict]]:
    """The launch configurations the verdict's optimisation set calls for."""
    out = [("default", dict(backend="default"))]
    if v.potential:
        part = v.partition or "row"
        # CLU + TOT: clustering in the probed partition, active agents 1..max
        for a in range(1, max_agents + 1):
            out.append((f"CLU-{part}+TOT{a}", dict(backend="agent", order=part, active_agents=a)))
        # the other partition at full agents: on B200 the reduced-size probe's
        # partition signal is often within noise (R22)
        alt = "col" if part == "row" else "row"
        out.append((f"CLU-{alt}", dict(backend="agent", order=alt)))
        # persistence + prefetch in the hardware order (no clustering): on B200
        # a single global wavefront can beat per-SM bands on DRAM page locality
        out.append(("PFH-identity", dict(backend="identity")))
        if has_staging and "BPS" in v.optimizations:
            # BPS: streaming operand bypasses L1 (TMA / no_allocate) vs through it
            out.append((f"CLU-{part}+L1", dict(backend="agent", order=part, staging="l1")))
            out.append((f"CLU-{part}+direct", dict(backend="agent", order=part, staging="direct")))
    else:
        # PFH with the reshaped (row) order: the agent's ring prefetches the
        # next tasks' operands; ring depth = prefetch distance
        for s in (1, 2, 4):
            out.append((f"PFH-row-s{s}", dict(backend="agent", order="row", stages=s)))
        out.append(("PFH-identity", dict(backend="identity")))
        for a in range(1, max_agents + 1):
            out.append((f"PFH-row+TOT{a}", dict(backend="agent", order="row", active_agents=a)))
    return out


@dataclass
class TuneResult:
    best: str
    best_kw: dict
    best_ms: float
    default_ms: float
    table: list[tuple[str, float]]

    @property
    def speedup(self) -> float:
        return self.default_ms / self.best_ms


def tune(run: Callable[..., object], cands: list[tuple[str, dict]], reps: int = 10,
         timer: Callable[[Callable[[], object], int], float] | None = None) -> TuneResult:
    """Time every candidate (run(**kw) launches it) and return the fastest."""
    timer = timer or (lambda fn, r: time_ms(fn, r))
    table = []
    for name, kw in cands:
        table.append((name, timer(lambda kw=kw: run(**kw), reps)))
    best = min(table, key=lambda t: t[1])
    dflt = next(ms for n, ms in table if n == "default")
    return TuneResult(best[0], dict(cands[[n for n, _ in cands].index(best[0])][1]), best[1], dflt, table)
