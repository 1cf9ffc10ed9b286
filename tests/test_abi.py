"""CPU-only checks of the C ABI: the library loads without a GPU, exports every
symbol include/ctaclust.h declares, its struct layouts match the binding, and
its host-only planner equals the independent oracle partition bit for bit."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

from oracle import plan as OP
from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ctaclust.h")


def header_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(cc_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_what_binding_lists():
    assert header_functions() == sorted(cc.EXPORTS)


def test_library_exports_every_declared_symbol():
    out = subprocess.check_output(["nm", "-D", "--defined-only", cc.LIB_PATH], text=True)
    syms = {ln.split()[-1] for ln in out.splitlines() if ln.strip()}
    missing = [f for f in header_functions() if f not in syms]
    assert not missing, missing
    L = cc.lib()
    assert cc.version().startswith("libctaclust")
    assert L.cc_status_string(-3) == b"user order is not a permutation"


LAYOUT_C = r"""
#include <stdio.h>
#include <stddef.h>
#include "ctaclust.h"
#define S(T) printf(#T " %zu\n", sizeof(T));
#define O(T, f) printf(#T "." #f " %zu\n", offsetof(T, f));
int main(void) {
  S(cc_plan_desc) O(cc_plan_desc, user_order) O(cc_plan_desc, device)
  S(cc_launch_opts) O(cc_launch_opts, d_census) O(cc_launch_opts, d_map) O(cc_launch_opts, l2_hint) O(cc_launch_opts, carveout)
  S(cc_matvec_args) O(cc_matvec_args, y) S(cc_atax_args) O(cc_atax_args, y)
  S(cc_bicg_args) O(cc_bicg_args, s) S(cc_mvt_args) O(cc_mvt_args, x2)
  S(cc_jacobi5_args) O(cc_jacobi5_args, result_is_b) O(cc_jacobi5_args, row_hi) S(cc_conv2d_args) O(cc_conv2d_args, w)
  S(cc_spmv_args) O(cc_spmv_args, part) O(cc_spmv_args, nnz) O(cc_spmv_args, xh) O(cc_spmv_args, n_hot)
  S(cc_hist64_args) O(cc_hist64_args, n) O(cc_hist64_args, counts)
  S(cc_jacobi5_halo_args) O(cc_jacobi5_halo_args, sweep0) O(cc_jacobi5_halo_args, ll)
  O(cc_jacobi5_halo_args, dn_ll) O(cc_jacobi5_halo_args, status)
  return 0;
}
"""


def test_struct_layouts_match_binding(tmp_path):
    src = tmp_path / "layout.c"
    src.write_text(LAYOUT_C)
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), "-o", str(exe), str(src)])
    got = dict(ln.rsplit(" ", 1) for ln in subprocess.check_output([str(exe)], text=True).splitlines())
    py = {"cc_plan_desc": cc.PlanDesc, "cc_launch_opts": cc.LaunchOpts, "cc_matvec_args": cc.MatvecArgs,
          "cc_atax_args": cc.AtaxArgs, "cc_bicg_args": cc.BicgArgs, "cc_mvt_args": cc.MvtArgs,
          "cc_jacobi5_args": cc.Jacobi5Args, "cc_conv2d_args": cc.Conv2dArgs, "cc_spmv_args": cc.SpmvArgs,
          "cc_hist64_args": cc.Hist64Args, "cc_jacobi5_halo_args": cc.Jacobi5HaloArgs}
    for key, val in got.items():
        if "." in key:
            t, f = key.split(".")
            f = {"w": "w"}.get(f, f)
            assert getattr(py[t], f).offset == int(val), key
        else:
            assert ctypes.sizeof(py[key]) == int(val), key


# ---- host-only planner vs the oracle ----------------------------------------
@pytest.mark.parametrize("order", ["row", "col", "tile"])
def test_planner_matches_oracle_tiny_grids(order):
    o = cc.ORDERS[order]
    for gx in range(1, 9):
        for gy in range(1, 9):
            for M in (1, 2, 3, 7, gx * gy, gx * gy + 3):
                p = cc.Plan(gx, gy, order, num_clusters=M, tile=(3, 2), device=None)
                perm, off = p.table()
                ref = OP.plan(gx, gy, o, M, 3, 2)
                assert np.array_equal(perm, ref["perm"]) and np.array_equal(off, ref["offsets"])
                assert (p.q, p.r) == (ref["q"], ref["r"])
                V = gx * gy
                for v in range(V):
                    w, i = p.lookup(v)
                    assert (w, i) == OP.f(V, M, v)
                    assert p.invert(w, i) == v


@pytest.mark.parametrize("gx,gy,order,tile,M", [
    (32, 32, "row", (1, 1), 148),        # config 1 matvec grid
    (64, 512, "col", (1, 1), 148),       # config 2 ATAX-family grid (n = 16384, 32x256 tiles)
    (512, 512, "tile", (8, 8), 148),     # config 3 Jacobi grid
    (256, 256, "tile", (4, 4), 148),     # config 4 conv grid
    (300, 7, "tile", (8, 3), 37),        # ragged tiles
])
def test_planner_matches_oracle_config_grids(gx, gy, order, tile, M):
    p = cc.Plan(gx, gy, order, num_clusters=M, tile=tile, device=None)
    perm, off = p.table()
    ref = OP.plan(gx, gy, cc.ORDERS[order], M, *tile)
    assert np.array_equal(perm, ref["perm"]) and np.array_equal(off, ref["offsets"])


def test_planner_user_order_and_errors():
    rng = np.random.default_rng(0)
    u = rng.permutation(35).astype(np.int32)
    p = cc.Plan(7, 5, "user", num_clusters=4, user_order=u, device=None)
    perm, off = p.table()
    ref = OP.plan(7, 5, OP.USER, 4, user_order=u)
    assert np.array_equal(perm, ref["perm"]) and np.array_equal(off, ref["offsets"])
    bad = u.copy()
    bad[3] = bad[4]
    with pytest.raises(cc.CtaclustError) as e:
        cc.Plan(7, 5, "user", num_clusters=4, user_order=bad, device=None)
    assert e.value.status == -3
    with pytest.raises(cc.CtaclustError) as e:
        cc.Plan(70000, 70000, "row", num_clusters=4, device=None)
    assert e.value.status == -2
    with pytest.raises(cc.CtaclustError) as e:
        cc.Plan(-1, 4, "row", num_clusters=4, device=None)
    assert e.value.status == -1
    with pytest.raises(cc.CtaclustError) as e:
        cc.Plan(4, 4, "tile", num_clusters=4, tile=(0, 2), device=None)
    assert e.value.status == -1
    with pytest.raises(cc.CtaclustError) as e:
        cc.Plan(4, 4, "row", num_clusters=0, device=None)        # M = 0 needs a device
    assert e.value.status == -1
    p = cc.Plan(4, 4, "row", num_clusters=3, device=None)
    with pytest.raises(cc.CtaclustError):
        p.lookup(16)
    with pytest.raises(cc.CtaclustError):
        p.invert(5, 2)                                           # cluster 2 has 5 slots: w <= 4
    with pytest.raises(cc.CtaclustError) as e:                   # host-only plan cannot launch
        cc._check(cc.lib().cc_launch(p.handle, 0, ctypes.byref(cc.CensusArgs(4, 4)), None, None, None))
    assert e.value.status == -7
    for bad in (dict(l2_hint=8), dict(l2_hint=-1), dict(carveout=101), dict(carveout=-2)):
        with pytest.raises(cc.CtaclustError) as e:               # options are validated first
            cc._check(cc.lib().cc_launch(p.handle, 0, ctypes.byref(cc.CensusArgs(4, 4)),
                                         ctypes.byref(cc.make_opts(**bad)), None, None))
        assert e.value.status == -1, bad


def test_empty_grid_and_more_clusters_than_ctas():
    p = cc.Plan(0, 5, "row", num_clusters=4, device=None)
    perm, off = p.table()
    assert p.V == 0 and list(off) == [0, 0, 0, 0, 0]
    p = cc.Plan(2, 2, "col", num_clusters=9, device=None)      # reading R8: surplus clusters empty
    perm, off = p.table()
    assert list(off) == [0, 1, 2, 3, 4, 4, 4, 4, 4, 4]


def test_kernel_grid():
    assert cc.kernel_grid("matvec", cc.MatvecArgs(None, 1024, 1024, 1024, None, None)) == (32, 32)
    assert cc.kernel_grid("bicg", cc.BicgArgs(None, 16384, 16384, 16384)) == (64, 512)
    assert cc.kernel_grid("atax", cc.AtaxArgs(None, 1004, 1001, 1001)) == (4, 32)
    assert cc.kernel_grid("jacobi5", cc.Jacobi5Args(None, None, 16384, 16384, 16384, 1)) == (512, 512)
    assert cc.kernel_grid("conv2d", cc.Conv2dArgs(None, None, 8192, 8192, 8192, 3)) == (256, 256)
    # jacobi5_wave (R34): 64-row tiles, 120-column strips for fuse <= 4, 112 for 5..8
    J = cc.Jacobi5Args
    assert cc.kernel_grid("jacobi5_wave", J(None, None, 16384, 16384, 16384, 100, None, 0, 0, 4)) == (137, 256)
    assert cc.kernel_grid("jacobi5_wave", J(None, None, 16384, 16384, 16384, 100, None, 0, 0, 8)) == (147, 256)
    assert cc.kernel_grid("jacobi5_wave", J(None, None, 128, 65, 120, 1, None, 0, 0, 0)) == (1, 2)
    with pytest.raises(cc.CtaclustError):
        cc.kernel_grid("jacobi5_wave", J(None, None, 128, 64, 64, 1, None, 0, 0, 9))
    assert cc.kernel_grid("jacobi5_wave", J(None, None, 16384, 16384, 16384, 100, None, 0, 0, 8, 256)) == (147, 64)
    assert cc.kernel_grid("jacobi5_wave", J(None, None, 16384, 1000, 16384, 100, None, 0, 0, 8, 16)) == (147, 63)
    with pytest.raises(cc.CtaclustError):
        cc.kernel_grid("jacobi5_wave", J(None, None, 128, 64, 64, 1, None, 0, 0, 8, 4))
    a = cc.SpmvArgs(1 << 24, 1 << 24, 1 << 28)
    assert cc.kernel_grid("spmv", a) == (((1 << 24) + (1 << 28) + 4095) // 4096, 1)
    assert cc.kernel_grid("hist64", cc.Hist64Args(None, 1 << 30, None)) == (32768, 1)
    assert cc.kernel_grid("hist64", cc.Hist64Args(None, 32769, None)) == (2, 1)
    assert cc.kernel_grid("hist64", cc.Hist64Args(None, 0, None)) == (0, 1)
    with pytest.raises(cc.CtaclustError):
        cc.kernel_grid("hist64", cc.Hist64Args(None, 1 << 32, None))


def test_kernel_ids_match_header():
    """cc_kernel enum values and CC_SPMV_SHUB_SLOTS as the binding mirrors them"""
    import re
    h = open(HEADER).read()
    ids = {m.group(1).lower(): int(m.group(2)) for m in re.finditer(r"\bCC_K_(\w+) = (\d+)", h)}
    assert ids == cc.KERNELS
    assert int(re.search(r"#define CC_SPMV_SHUB_SLOTS (\d+)", h).group(1)) == cc.SPMV_SHUB_SLOTS


def test_arg_structs_own_their_host_buffers():
    """jacobi5_args' result_is_b flag and conv2d_args' filter are host memory
    the library reads or writes at launch: the struct must keep them alive
    even when the caller keeps only the struct (`jacobi5_args(...)[0]`; a
    dropped flag was a use-after-free that crashed sharded runs)."""
    import gc
    import torch
    a = torch.zeros(8, 8)
    args = cc.jacobi5_args(a, a, 1)[0]
    gc.collect()
    assert ctypes.addressof(args._keep) == args.result_is_b
    c = cc.conv2d_args(a, a, np.ones((3, 3)))[0]
    gc.collect()
    assert c._keep.ctypes.data == c.w
    h = cc.jacobi5_halo_args(a, a, 1)[0]
    assert ctypes.addressof(h._keep) == h.result_is_b


def test_in_out_share_leading_dimension():
    """The C ABI carries one leading dimension for a kernel's input and output
    (cc_conv2d_args.ld, cc_jacobi5_args.ld): the binding refuses a pair whose
    strides differ instead of writing the output with the input's pitch."""
    import torch
    a = torch.zeros(8, 72)[:, :70]
    b = torch.zeros(8, 70)
    with pytest.raises(cc.CtaclustError):
        cc.conv2d_args(a, b, [[1.0]])
    with pytest.raises(cc.CtaclustError):
        cc.jacobi5_args(a, b, 1)
    cc.conv2d_args(a, torch.zeros(8, 72)[:, :70], [[1.0]])
