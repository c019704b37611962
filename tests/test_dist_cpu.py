"""The N>1 launch path of bench.py on CPU (gloo, world_size 2, 127.0.0.1): rendezvous from
the torchrun environment variables, barriers, max-over-ranks timing, sums of the per-rank
byte counters, the host matrices shared by the rank-mode processes (rank 0 generates them
into /dev/shm file mappings, every rank sees the same bits), and the rule that only rank 0
prints.  The data path itself has no collective: the fan-out of tiles is the library's
peer forwarding."""
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

WORKER = r"""
import os, sys, json
sys.path.insert(0, %(root)r)
import bench
rank, ws = bench.dist_setup("gloo")
assert ws == 2 and rank == int(os.environ["RANK"])
bench.barrier(ws)
mx = bench.max_over_ranks(10.0 + rank, ws)
assert mx == 11.0, mx
assert bench.sum_over_ranks([1.0 + rank, 5.0], ws) == [3.0, 10.0]
# rank-mode host matrices: one generator run on rank 0, the same bits on every rank
import numpy as np, inputs
A, B, C, paths, base = bench.share_inputs(48, rank, ws)
assert np.array_equal(np.asarray(B), inputs.uniform(inputs.SEED_B, 48, 48))
assert A.shape == (48, 48) and np.asfortranarray(A).flags.f_contiguous
assert base and base.startswith(("/dev/shm", "/tmp"))  # session files: base + ".session<n>"
assert len(paths) == (0 if os.environ.get("XK_SHARE") == "memfd" else 3)
# per-GPU values gathered in rank order (per-GPU H2D bytes of the ablation)
assert bench.gather_per_gpu(7.0 + rank, ws) == [7.0, 8.0]
bench.barrier(ws)
if rank == 0:
    for p in paths:
        os.unlink(p)
# reference arm under torchrun: rank 0 alone prints one JSON line, the other exits quietly
if rank == 0:
    print(json.dumps({"rank": 0, "max": mx}))
bench.barrier(ws)
import torch.distributed as dist
dist.destroy_process_group()
"""


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("share", ["shm", "memfd"])
def test_two_rank_gloo_barrier_and_max_timing(share):
    """share=memfd: the host matrices are anonymous memfds of rank 0 opened by rank 1
    through /proc/<pid>/fd (the fallback when /dev/shm is too small)."""
    port = free_port()
    procs = []
    for r in range(2):
        env = dict(os.environ, RANK=str(r), LOCAL_RANK=str(r), WORLD_SIZE="2", MASTER_ADDR="127.0.0.1",
                   MASTER_PORT=str(port), XK_SHARE=share)
        procs.append(subprocess.Popen([sys.executable, "-c", WORKER % {"root": ROOT}], env=env,
                                      stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True))
    outs = [p.communicate(timeout=120) for p in procs]
    for p, (o, e) in zip(procs, outs):
        assert p.returncode == 0, e
    assert '"max": 11.0' in outs[0][0]
    assert outs[1][0].strip() == ""  # only rank 0 prints


def test_reference_arm_nonzero_ranks_exit_quietly():
    """bench.py --impl reference under a 2-rank launch: rank 1 does no work and prints nothing."""
    port = free_port()
    env = dict(os.environ, RANK="1", LOCAL_RANK="1", WORLD_SIZE="2", MASTER_ADDR="127.0.0.1",
               MASTER_PORT=str(port), XK_DIST_BACKEND="gloo")
    # rank 1 alone would wait for rank 0 at the rendezvous; run both
    env0 = dict(env, RANK="0", LOCAL_RANK="0")
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1", "--warmup", "0",
           "--n", "256"]
    p0 = subprocess.Popen(cmd, env=env0, stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True)
    p1 = subprocess.Popen(cmd, env=env, stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True)
    o0, e0 = p0.communicate(timeout=300)
    o1, e1 = p1.communicate(timeout=300)
    assert p0.returncode == 0, e0
    assert p1.returncode == 0, e1
    assert '"impl": "reference"' in o0 and o1.strip() == ""
