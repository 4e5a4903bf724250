"""The N > 1 path on the one-GPU box: 2 processes (torchrun), CUDA IPC
between them, bootstrap over gloo; results vs the oracle.  The two processes
time-slice the GPU, so this checks correctness of the cross-process path, not
its speed."""
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_two_processes_ipc(tmp_path):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=29611", os.path.join(ROOT, "tests", "mp_worker.py"),
           str(tmp_path)]
    p = subprocess.run(cmd, capture_output=True, text=True, timeout=400)
    assert p.returncode == 0, p.stdout[-3000:] + p.stderr[-3000:]
    res = [np.load(os.path.join(tmp_path, f"rank{r}.npz")) for r in range(2)]
    Np, L = 3, 1000
    x = np.stack([synth.normal_f32(synth.BASE_SEED, r, 0, Np * L) for r in range(2)])
    for name, algo in (("ring", oracle.RING), ("rd", oracle.RD), ("direct", oracle.DIRECT),
                       ("direct_push", oracle.DIRECT), ("ll", oracle.DIRECT)):
        ref, _, _ = oracle.pallreduce(x, Np, algo)
        for r in range(2):
            np.testing.assert_array_equal(res[r][name].view(np.uint32), ref[r].view(np.uint32))
            for e in range(3):  # pc_epoch_all epochs across processes
                np.testing.assert_array_equal(res[r][f"{name}_epoch_all{e}"].view(np.uint32),
                                              ref[r].view(np.uint32))
    # INLINE allreduce across processes (R33): the DIRECT bits (O6), 3 epochs
    Np, L = 5, 777
    x = np.stack([synth.normal_f32(synth.BASE_SEED + 3, r, 0, Np * L) for r in range(2)])
    ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
    for r in range(2):
        for e in range(3):
            np.testing.assert_array_equal(res[r]["inline%d" % e].view(np.uint32), ref[r].view(np.uint32))
    # overlap across processes: partition 0 completed inside each producer
    Np, L = 4, 4099
    x = np.stack([synth.normal_f32(synth.BASE_SEED + 4, r, 0, Np * L) for r in range(2)])
    ref, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
    for r in range(2):
        np.testing.assert_array_equal(res[r]["overlap"].view(np.uint32), ref[r].view(np.uint32))
        s = res[r]["overlap_stamps"][0]
        assert 0 < s[2] < s[3], s
    n = 2048 * 8
    a = synth.uniform_f32(synth.BASE_SEED, 0, 0, n)
    b = synth.uniform_f32(synth.BASE_SEED, 0, 1, n)
    consumed, arr = oracle.p2p(((a + b).astype(np.float32)).view(np.uint8)[None], 8, 2,
                               np.arange(8, dtype=np.int32)[None])
    assert (arr == 1).all()
    np.testing.assert_array_equal(res[1]["p2p"].view(np.uint8), consumed[0])
    a2 = synth.uniform_f32(synth.BASE_SEED, 1, 0, n)
    np.testing.assert_array_equal(res[0]["p2p_engine"], (a2 + a2).astype(np.float32))
    a3 = synth.uniform_f32(synth.BASE_SEED, 0, 7, 2048 * 2)
    np.testing.assert_array_equal(res[1]["p2p_ll"], (a3 + a3).astype(np.float32))
    # Jacobi: each process holds its own block; together they equal the oracle
    ref = oracle.jacobi_seq(synth.jacobi_init(256, 256, "random"), 30)
    np.testing.assert_array_equal(res[0]["jacobi"][:128], ref[:128])
    np.testing.assert_array_equal(res[1]["jacobi"][128:], ref[128:])
