"""Host nm_reorder vs nm_reorder_gpu (Stage-1 + counts on the device) on larger graphs: wall
time and bit-identity of the two permutations.  usage: python tools/reorder_timing.py [out.jsonl]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ppopp_chensz0s25_b200 import api, graphs  # noqa: E402

CASES = [("band", 262144, 16, 64, 8, 2), ("band", 1048576, 16, 128, 16, 1),
         ("pl", 262144, 16, 128, 16, 1), ("pl", 65536, 16, 64, 8, 1)]


def main():
    out = open(sys.argv[1], "w") if len(sys.argv) > 1 else None
    torch.cuda.init()
    for kind, n, d, V, M, outer in CASES:
        if kind == "band":
            ip, ic = graphs.banded_graph(n, d, 21)
        else:
            ip, ic = graphs.lmcl_graph(n, n * d // 2, 2.1, 1, 0.0, 21, scramble=True)
        t = time.time()
        pg, sg = api.reorder(ip, ic, V, 2, M, max_outer=outer, device=True)
        tg = time.time() - t
        t = time.time()
        ph, sh = api.reorder(ip, ic, V, 2, M, max_outer=outer)
        th = time.time() - t
        rec = {"graph": kind, "n": n, "nnz": int(len(ic)), "V": V, "M": M, "max_outer": outer,
               "host_s": th, "gpu_s": tg, "identical": bool((pg == ph).all()),
               "stage1_iters": sg["stage1_iters"], "mb": [sg["mb_init"], sg["mb_final"]],
               "omega": [sg["omega_init"], sg["omega_final"]]}
        print(json.dumps(rec), flush=True)
        if out:
            out.write(json.dumps(rec) + "\n")
            out.flush()


if __name__ == "__main__":
    main()
