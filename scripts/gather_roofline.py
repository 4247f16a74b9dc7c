"""Random-gather roofline: sustained 32-byte-sector rate for buffers that fit
in L2 (64 MB), the C1 working set (~450 MB: col + filter + edge set) and HBM (2 GB), with 1-8
dependent chains in flight per thread."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_journals_pacmmod_yelsg24_b200 as G  # noqa: E402

with G.Context(0) as ctx:
    for mb in (64, 450, 2048):
        for inflight in (1, 2, 4, 8):
            r = ctx.gather_roofline(mb << 20, inflight)
            print(json.dumps({"buffer_mb": mb, "inflight": inflight, "sectors_per_s": r, "GBps": r * 32 / 1e9}),
                  flush=True)
