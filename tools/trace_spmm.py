"""Timeline of the SpMM pipeline on CTA 0 (profiling aid, not part of the product).

Runs the bench workload once with NM_SPMM_TRACE set: the kernel records clock64() at the
hand-off points of its first 1024 chunks / units and this script prints per-chunk latencies:
  rec   : record producer passes the empty-barrier (stage free) and issues the bulk copy
  ld    : loader thread 0 sees the record landed (full_a)
  ldone : loader thread 0 finished issuing gathers + metadata
  mma   : MMA warp sees the stage ready (full_b)
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch

    import bench
    from paper_conf_ppopp_chensz0s25_b200 import api, graphs
    wl = sys.argv[1] if len(sys.argv) > 1 else bench.DEFAULT
    w = bench.parse_workload(wl)
    ip, ic, vals, X32 = bench.make_graph(w)
    perm, _ = api.reorder(ip, ic, w["V"], 2, w["M"])
    tau = w["tau"] if w["tau"] is not None else api.hybrid_tau(w["F"])
    P = api.pack(ip, ic, perm, w["V"], 2, w["M"], dtype=w["dtype"], val=vals, order="original", tau=tau)
    xb, _ = graphs.round16(X32, w["dtype"])
    X = torch.from_numpy(xb.view(np.int16)).cuda().view(torch.float16)
    Y = torch.empty((w["n"], w["F"]), device="cuda")
    for _ in range(3):
        api.spmm(P, X, Y, part="sptc")
    torch.cuda.synchronize()
    path = "/tmp/nm_trace.bin"
    os.environ["NM_SPMM_TRACE"] = path
    api.spmm(P, X, Y, part="sptc")
    torch.cuda.synchronize()
    del os.environ["NM_SPMM_TRACE"]
    t = np.fromfile(path, dtype=np.uint64).astype(np.int64)
    if os.environ.get("NM_TRACE_SAVE"):
        np.save(os.environ["NM_TRACE_SAVE"], t)
    full = t[:8192].reshape(1024, 8)
    ch = full[:, :4]
    un = t[8192:].reshape(2048, 4)
    n = int((ch[:, 3] > 0).sum())  # chunks the MMA issued (the producer marks sub-batches only)
    ch = ch[:n]
    base = ch[0, 0]
    ch[:, 0] = np.where(ch[:, 0] > 0, ch[:, 0], 0)
    ch[:, 0] = np.maximum.accumulate(ch[:, 0])  # issue time of the sub-batch holding the chunk
    # loader sub-steps (slots 1 -> 4 -> 5 -> 6 -> 7 -> 2): sees record, gathers issued, record
    # expanded + released, A tile + tcgen05.st issued, tcgen05.wait::st done, arrived
    sub = full[:n][:, [7, 1, 4, 5, 6, 2]]
    own = sub[:, 0] > 0
    if own.any():
        d = np.diff(sub[own], axis=1)
        for name, v in zip(["stage free -> record seen", "gathers issue", "expand+release",
                            "A sts + tcgen05.st", "wait::st+fence+arrive"], d.T):
            print("loader %-22s median %6d  p90 %6d cycles" % (name, np.median(v), np.percentile(v, 90)))
    G = int(os.environ.get("NM_TRACE_GROUPS", "3"))
    f = full[:n].astype(np.int64)
    if n > 2 * G:
        ws = f[G:, 7] - f[:-G, 2]   # own previous chunk arrived -> this chunk's stage free
        wr = f[G:, 1] - f[G:, 7]    # stage free -> record landed
        busy = f[G:, 2] - f[G:, 1]  # record landed -> arrive (loader work)
        for name, v in [("loader wait for stage", ws), ("loader wait for record", wr), ("loader busy", busy)]:
            print("%-30s mean %6.0f median %6d p90 %6d cycles" % (name, v.mean(), np.median(v), np.percentile(v, 90)))
    sbt = t[12288:].reshape(1024, 4)
    nsb = int((sbt[:, 0] > 0).sum())
    if nsb > 1:
        sbt = sbt[:nsb]
        wait_space = sbt[:, 1] - sbt[:, 0]
        other = sbt[1:, 0] - sbt[:-1, 1]
        infl, ringb = sbt[:, 2] >> 32, sbt[:, 2] & 0xFFFFFFFF
        nw, m = sbt[:, 3] >> 32, sbt[:, 3] & 0xFFFFFFFF
        print("producer: %d sub-batches (mean %.1f records), ring-space wait mean %.0f (p90 %.0f), other work "
              "between waits mean %.0f (p90 %.0f) cycles; at entry: descriptors in flight mean %.1f, ring bytes "
              "mean %.0f; descriptor waits per sub-batch mean %.2f" %
              (nsb, m.mean(), wait_space.mean(), np.percentile(wait_space, 90), other.mean(),
               np.percentile(other, 90), infl.mean(), ringb.mean(), nw.mean()))
    ch = ch - base
    print("chunks traced:", n)
    d_rec_ld = ch[:, 1] - ch[:, 0]
    d_ld = ch[:, 2] - ch[:, 1]
    d_ld_mma = ch[:, 3] - ch[:, 2]
    gap = np.diff(ch[:, 0])
    for name, v in [("record issue -> loader sees record", d_rec_ld), ("loader issue time", d_ld),
                    ("loader done -> MMA sees stage", d_ld_mma), ("record issue interval", gap),
                    ("MMA interval", np.diff(ch[:, 3]))]:
        print("%-38s median %7d  p10 %7d  p90 %7d cycles" % (name, np.median(v), np.percentile(v, 10),
                                                             np.percentile(v, 90)))
    mi = np.diff(ch[:, 3])
    print("MMA interval mean %.0f; share of time in gaps > 1000 cycles: %.2f" %
          (mi.mean(), mi[mi > 1000].sum() / mi.sum()))
    nu = int((un[:, 1] > 0).sum())
    un = un[:nu] - base
    # unit boundary cost: MMA start of unit k+1 minus the MMA time of unit k's last chunk
    print("epilogue start - MMA start (median): %.0f" % np.median(un[:, 2] - un[:, 1]))
    print("units traced:", nu)
    print("unit: mma_start(tempty ok) epi_start(tfull) epi_end")
    for k in range(min(8, nu)):
        print(k, un[k, 1], un[k, 2], un[k, 3])
    print("epilogue duration median", np.median(un[:, 3] - un[:, 2]))
    print("first 24 chunks (rec, ld, ldone, mma):")
    print(ch[:24])


if __name__ == "__main__":
    main()
