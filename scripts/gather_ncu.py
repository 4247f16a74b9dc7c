"""K5 random-gather launches at three buffer sizes, for an ncu capture of their DRAM bytes per
requested sector (is a random 32-byte sector fetched from HBM as one sector or as a larger atom?).
usage (on the GPU box): ncu --metrics ... python scripts/gather_ncu.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402

with G.Context(0) as ctx:
    for mb in (64, 128, 450, 2048):
        r = ctx.gather_roofline(mb << 20, 4)
        print(mb, "MB", r, "sectors/s", flush=True)
