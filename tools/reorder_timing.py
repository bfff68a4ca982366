"""nm_reorder (host Stage-1 + host Stage-2 gain tables) vs nm_reorder_gpu (Stage-1, the counts and
the Stage-2 gain tables on the device, the picks on the host): wall time, bit-identity of the two
permutations, violation removal -- on graphs shaped like the paper's workloads, compared with
Table 7's reordering times (0.01-30.55 s).
usage: python tools/reorder_timing.py [out.jsonl]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ppopp_chensz0s25_b200 import api, graphs  # noqa: E402

# (name, graph builder, V, M, reorder options, run the host version too)
CASES = [
    ("banded n=262k d=16", lambda: graphs.banded_graph(262144, 16, 21), 64, 8, dict(max_outer=2), True),
    ("banded n=1M d=16", lambda: graphs.banded_graph(1 << 20, 16, 21), 1, 4, dict(max_outer=1), True),
    ("power-law n=262k d=16", lambda: graphs.lmcl_graph(262144, 262144 * 8, 2.1, 1, 0.0, 21, scramble=True),
     1, 4, dict(max_outer=1), True),
    ("power-law n=65k d=16", lambda: graphs.lmcl_graph(65536, 65536 * 8, 2.1, 1, 0.0, 21, scramble=True),
     64, 8, dict(max_outer=1), True),
    ("C3 reddit 1:2:4, one Alg.1 iteration", lambda: graphs.gnn_graph("reddit"), 1, 4,
     dict(max_outer=0, max_stage2=0), True),
    ("C3 reddit 1:2:4, MAXITER = 10", lambda: graphs.gnn_graph("reddit"), 1, 4, dict(), False),
    ("C4 proteins 128:2:16, MAXITER = 10", lambda: graphs.gnn_graph("proteins"), 128, 16, dict(), False),
]


def main():
    out = open(sys.argv[1], "w") if len(sys.argv) > 1 else None
    torch.cuda.init()
    cache = {}
    for name, make, V, M, opts, host in CASES:
        key = name.split(",")[0].split(" 1:2")[0]
        if key not in cache:
            cache = {key: make()}
        ip, ic = cache[key]
        t = time.time()
        pg, sg = api.reorder(ip, ic, V, 2, M, device=True, **opts)
        tg = time.time() - t
        rec = {"graph": name, "n": int(len(ip) - 1), "nnz": int(len(ic)), "V": V, "M": M, "opts": opts, "gpu_s": tg,
               "omega": [sg["omega_init"], sg["omega_final"]], "mb": [sg["mb_init"], sg["mb_final"]],
               "outer_iters": sg["outer_iters"], "stage1_iters": sg["stage1_iters"],
               "stage2_passes": sg["stage2_passes"],
               "violation_removal": None if sg["omega_init"] == 0 else 1 - sg["omega_final"] / sg["omega_init"]}
        if host:
            t = time.time()
            ph, sh = api.reorder(ip, ic, V, 2, M, **opts)
            rec["host_s"] = time.time() - t
            rec["identical"] = bool((pg == ph).all())
        print(json.dumps(rec), flush=True)
        if out:
            out.write(json.dumps(rec) + "\n")
            out.flush()


if __name__ == "__main__":
    main()
