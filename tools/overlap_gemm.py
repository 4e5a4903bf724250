"""Producer/collective overlap with a COMPUTE-bound producer (a6 / NEXT-2
context): every virtual rank computes its bf16 "gradient" with GEMMs, bucket by
bucket (cuBLAS, the user's computation), and allreduces it with one
partitioned-allreduce request per bucket (DIRECT, bf16 SUM).
  serial:   every bucket's GEMM, then every bucket's allreduce
  overlap:  after bucket k's GEMM the host Preadies bucket k (pc_pready_range
            on the compute stream) and waits on a communication stream, so
            bucket k's engine — forked at that Pready, full width, on the
            library's high-priority stream — reduces while GEMM k+1 runs.
JSON lines: ms per step (CUDA events), busBW of the allreduce part."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import torch  # noqa: E402

import paper_conf_sc_temucinslsga24_b200 as pc  # noqa: E402


def run(P, buckets, M, N, K, reps=10):
    g, cs = pc.local_comms(P, 0)
    torch.manual_seed(0)
    comp, commst = torch.cuda.Stream(), torch.cuda.Stream()
    # bucket k of every rank in one batched GEMM: A[k] (P, M, K) x B (P, K, N) -> grad[k] (P, M*N)
    A = [torch.randn(P, M, K, device="cuda", dtype=torch.bfloat16) for _ in range(buckets)]
    B = torch.randn(P, K, N, device="cuda", dtype=torch.bfloat16)
    grad = torch.empty(buckets, P, M * N, device="cuda", dtype=torch.bfloat16)
    out = torch.empty(P, buckets, M * N, device="cuda", dtype=torch.bfloat16)
    Np = 8  # partitions per bucket
    reqs = [[pc.pallreduce_init(grad[k, r], out[r, k], Np, M * N // Np, pc.BF16, pc.SUM, pc.ALGO_DIRECT, cs[r])
             for r in range(P)] for k in range(buckets)]
    for k in range(buckets):
        for q in reqs[k]:
            q.start(comp)
        pc.run_ranks([(lambda q=q: q.pbuf_prepare(comp)) for q in reqs[k]])
        pc.preadyall(reqs[k], comp)
        for q in reqs[k]:
            q.wait_on_stream(comp)
    torch.cuda.synchronize()

    def gemm(k):
        with torch.cuda.stream(comp):
            torch.bmm(A[k], B, out=grad[k].view(P, M, N))

    def serial():
        for k in range(buckets):
            gemm(k)
        for k in range(buckets):
            pc.epoch_all(reqs[k], pready=True, stream=comp)
            for q in reqs[k]:
                q.wait_on_stream(comp)

    def overlap():
        ev = torch.cuda.Event()
        for k in range(buckets):
            pc.startall(reqs[k], comp)
            pc.pbuf_prepare_all(reqs[k], comp)
        for k in range(buckets):
            gemm(k)
            pc.preadyall(reqs[k], comp)  # every partition of bucket k: the engine forks here, full width
            ev.record(comp)
            commst.wait_event(ev)
            for q in reqs[k]:
                q.wait_on_stream(commst)
        comp.wait_stream(commst)

    def gemm_only():
        for k in range(buckets):
            gemm(k)

    def comm_only():
        for k in range(buckets):
            pc.epoch_all(reqs[k], pready=True, stream=comp)
            for q in reqs[k]:
                q.wait_on_stream(comp)

    res = {}
    for name, fn in (("gemm_only", gemm_only), ("comm_only", comm_only), ("serial", serial), ("overlap", overlap)):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(comp)
        for _ in range(reps):
            fn()
        e1.record(comp)
        torch.cuda.synchronize()
        res[name] = e0.elapsed_time(e1) / reps
    errs = [q.error() for row in reqs for q in row if q.error()[0] != 0]
    # parity (sampled): the overlapped result equals the serial one bit for bit
    overlap()
    torch.cuda.synchronize()
    o1 = [out.clone()]
    serial()
    torch.cuda.synchronize()
    same = torch.equal(o1[0], out)
    for row in reqs:
        for q in row:
            q.free()
    for c in cs:
        c.destroy()
    g.destroy()
    S = buckets * M * N * 2
    print(json.dumps({"P": P, "buckets": buckets, "M": M, "N": N, "K": K, "bytes_per_rank": S, **res,
                      "overlap_speedup": res["serial"] / res["overlap"], "errors": errs, "overlap_equals_serial": same}),
          flush=True)


if __name__ == "__main__":
    torch.cuda.set_device(0)
    for K in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "512,1024,2048,4096").split(",")]:
        run(8, 8, 2048, 1536, K)
