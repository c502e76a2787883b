"""Write tests/golden/oracle_digests.json: per-level digests of the ORACLE's
hierarchy for the BASELINE.json configs.  Calls only graphgen/ (inputs) and
oracle/ (results) — never the CUDA path — so the stored values are oracle
values.  GPU parity tests compare the CUDA hierarchy's
digests against these at full size.

usage: python tests/golden/make_digests.py [config ...]   (default: 1 2 3 4)
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import graphgen as gg  # noqa: E402
import oracle as o     # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "oracle_digests.json")


def level_digest(lv):
    c = lv.graph
    return dict(n_c=lv.n_c, nnz_c=c.nnz, sum_wc=int(c.wgt.astype(np.int64).sum()),
                intra=int(c.intra), sha_M=gg.sha16(lv.M), sha_G=gg.sha16(c.row_ptr, c.col, c.wgt),
                sha_vwgt=gg.sha16(c.vwgt), t_map_s=round(lv.t_map, 3), t_build_s=round(lv.t_build, 3))


def main(cfgs):
    data = json.load(open(OUT)) if os.path.exists(OUT) else {}
    for k in cfgs:
        c = gg.CONFIGS[k]
        t0 = time.time()
        g = gg.config(k)
        tg = time.time() - t0
        H = o.hierarchy(g, c["cutoff"], gg.COARSEN_SEED)
        data[str(k)] = dict(
            name=c["name"], cutoff=c["cutoff"], seed=gg.COARSEN_SEED, n=g.n, nnz=g.nnz,
            sha_G0=gg.sha16(g.row_ptr, g.col), levels=[level_digest(lv) for lv in H.levels],
            stop_reason=H.stop_reason, discarded_n_c=H.discarded_n_c,
            oracle_total_s=round(H.t_total, 3), gen_s=round(tg, 3))
        print(k, c["name"], g.n, g.nnz, [lv.n_c for lv in H.levels], H.stop_reason,
              f"oracle {H.t_total:.1f}s", flush=True)
        json.dump(data, open(OUT, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main([int(a) for a in sys.argv[1:]] or [1, 2, 3, 4])
