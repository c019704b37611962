"""Rank mode's host-side synchronisation on CPU (no GPU needed): the session file protocol
(rank 0 creates it, the others join, rank 0 removes it), the shared-memory barrier across
processes (every rank sees every arrival of a round before leaving it), and the abort rule
(a failing rank makes its peers' barriers fail instead of hanging).  DESIGN.md §8."""
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

WORKER = r"""
import json, sys
sys.path.insert(0, %(root)r)
import paper_conf_sc_gautierl21_b200 as xk
rc, seen = xk.session_selftest(%(path)r, %(rank)d, %(world)d, %(rounds)d, %(abort)d, 90.0)
print(json.dumps({"rc": rc, "seen": seen}))
"""


def run(world, rounds, abort_rank=-1, abort_at=-1):
    with tempfile.TemporaryDirectory() as d:
        path = os.path.join(d, "session")
        procs = [subprocess.Popen([sys.executable, "-c", WORKER % {
            "root": ROOT, "path": path, "rank": r, "world": world, "rounds": rounds,
            "abort": abort_at if r == abort_rank else -1}], stdout=subprocess.PIPE, stderr=subprocess.PIPE,
            text=True) for r in range(world)]
        outs = []
        for p in procs:
            o, e = p.communicate(timeout=120)
            assert p.returncode == 0, e
            import json
            outs.append(json.loads(o.strip().splitlines()[-1]))
        removed = not os.path.exists(path)
    return outs, removed


def test_barrier_rounds_across_processes():
    world, rounds = 4, 25
    outs, removed = run(world, rounds)
    for o in outs:
        assert o["rc"] == 0
        assert o["seen"] == [world] * rounds  # all arrivals of round r visible when leaving it
    assert removed, "rank 0 removes the session file"


def test_abort_fails_peers_instead_of_hanging():
    outs, _ = run(3, 6, abort_rank=2, abort_at=3)
    assert outs[2]["rc"] == 0, outs            # the aborting rank itself returns cleanly
    assert outs[0]["rc"] == 2 and outs[1]["rc"] == 2, outs  # XK_ERR_CUDA at the failed barrier
    assert outs[0]["seen"][:3] == [3, 3, 3] and outs[1]["seen"][:3] == [3, 3, 3]


def test_second_creator_refused():
    """A session path must be unique: rank 0 refuses an existing file (XK_ERR_CONFIG)."""
    import paper_conf_sc_gautierl21_b200 as xk
    with tempfile.TemporaryDirectory() as d:
        path = os.path.join(d, "session")
        open(path, "w").close()
        rc, _ = xk.session_selftest(path, 0, 1, 1, -1, 5.0)
        assert rc == 4
