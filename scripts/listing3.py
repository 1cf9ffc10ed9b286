#!/usr/bin/env python
"""Listing 3 on the GPU box: default and staggered runs -> JSON summary.
    python scripts/listing3.py gpurun_out/listing3.json"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_lis0l0c17_b200 import ctaclust as cc, microbench as mb  # noqa: E402


def main(out):
    info = cc.device_info()
    res = {"device": info, "slots": mb.SLOTS}
    for name, stagger, turns in [("default", 0, 2), ("default_4turn", 0, 4), ("staggered_1200", 1200, 2)]:
        mb.run(turnarounds=turns, stagger=stagger)                # warm-up launch
        smid, ticks = mb.run(turnarounds=turns, stagger=stagger)
        res[name] = mb.analyze(smid, ticks, num_sms=info["num_sms"])
        s0 = smid[0]
        on0 = [(int(b), int(t)) for b, (s, t) in enumerate(zip(smid, ticks)) if s == s0]
        res[name]["sm_of_cta0_all"] = on0
        print(name, {k: v for k, v in res[name].items() if k.startswith("ticks") or k.startswith("first_wave")})
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/listing3.json")
