"""One process of a rank-mode run (one process per GPU), spawned by
tests/test_gpu_rank.py: `world` copies of this script share one session file and host
matrices in shared file mappings, make the same collective calls, and each prints one JSON
line with its own GPU's byte counters.  Rank 0 checks the numbers against the CPU oracle
(test infrastructure: tests/ may use oracle/)."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import inputs  # noqa: E402
import paper_conf_sc_gautierl21_b200 as xk  # noqa: E402

EPS = 2.0 ** -53


def shared(args, name, rows, cols):
    return xk.shared_matrix(os.path.join(args.dir, name), rows, cols, create=args.rank == 0)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rank", type=int, required=True)
    ap.add_argument("--world", type=int, required=True)
    ap.add_argument("--session", required=True)
    ap.add_argument("--dir", required=True)
    ap.add_argument("--case", required=True)
    ap.add_argument("--n", type=int, default=1000)
    ap.add_argument("--tile", type=int, default=256)
    ap.add_argument("--probe", type=int, default=0)
    ap.add_argument("--arena", type=int, default=1 << 30)
    ap.add_argument("--topo", default="ranked")
    ap.add_argument("--optimistic", type=int, default=1)
    args = ap.parse_args()
    r, N, T = args.rank, args.n, args.tile
    out = {"rank": r, "case": args.case, "ok": True, "checks": []}

    def check(name, cond):
        out["checks"].append(name)
        if not cond:
            out["ok"] = False
            out.setdefault("failed", []).append(name)

    mats = {}

    def mat(name, rows, cols, fill=None):
        """Shared host matrix; rank 0 fills it before xk_init (collective), the others map
        it after, when the file is complete."""
        if r != 0:
            mats[name] = (rows, cols)
            return None
        M = shared(args, name, rows, cols)
        if fill is not None:
            fill(M)
            M.flush()
        mats[name] = M
        return M

    def reopen():
        for name, (rows, cols) in list(mats.items()):
            mats[name] = xk.shared_matrix(os.path.join(args.dir, name), rows, cols, create=False)

    if args.case in ("gemm", "compose", "dod", "distribute"):
        mat("A", N, N, lambda M: inputs.integers(1, N, N, out=M))
        mat("B", N, N, lambda M: inputs.integers(2, N, N, out=M))
        mat("C", N, N, lambda M: inputs.integers(3, N, N, out=M))
        mat("E", N, N, lambda M: M.fill(0.0))
        if args.case == "compose":
            mat("D", N, N, lambda M: M.fill(0.0))
    elif args.case == "big":
        mat("A", N, N, lambda M: inputs.integers(1, N, N, out=M))
        mat("B", N, N, lambda M: inputs.integers(2, N, N, out=M))
        mat("C", N, N, lambda M: inputs.integers(3, N, N, out=M))
    elif args.case == "blas3":
        k = N // 2 + 3
        mat("A", N, k, lambda M: inputs.integers(1, N, k, out=M))
        mat("B", N, k, lambda M: inputs.integers(2, N, k, out=M))
        mat("C", N, N, lambda M: inputs.integers(3, N, N, out=M))
        mat("S", N, N, lambda M: inputs.integers(4, N, N, out=M))
        mat("X", N, N, lambda M: inputs.integers(5, N, N, out=M))
        mat("L", N, N, lambda M: inputs.tri_dd(4, N, lower=True, out=M))
    keep = ("C",) if args.case == "big" else tuple(mats)
    C0 = {name: np.array(mats[name], order="F") for name in keep} if r == 0 else None

    if args.case == "mismatch":
        # rank 1 asks for another tile size: every rank must refuse (different plans)
        try:
            xk.init(rank=r, world=args.world, session=args.session, tile=T * (2 if r == 1 else 1),
                    probe=False, arena_bytes=args.arena)
            out["init_error"] = 0
            xk.finalize()
        except xk.XKError as e:
            out["init_error"] = e.code
        print(json.dumps(out), flush=True)
        return
    xk.init(rank=r, world=args.world, session=args.session, tile=T, probe=bool(args.probe),
            arena_bytes=args.arena, topo=args.topo, optimistic=bool(args.optimistic))
    if r != 0:
        reopen()
    for M in mats.values():
        xk.register(M)
    xk.reset_stats()
    m = mats
    if args.case == "gemm":
        # C <- -2 A B + 0.5 C (exact integers: any summation order gives the same bits)
        assert xk.dgemm("N", "N", N, N, N, -2.0, m["A"], N, m["B"], N, 0.5, m["C"], N) == 0
        # and a transposed call on the result
        assert xk.dgemm("T", "N", N, N, N, 1.0, m["A"], N, m["C"], N, 0.0, m["E"], N) == 0
    elif args.case == "compose":
        # D = A*B; E = D*C with no coherence in between: D is read from the
        # GPUs, never from the host; then E and D are made coherent
        assert xk.dgemm_async("N", "N", N, N, N, 1.0, m["A"], N, m["B"], N, 0.0, m["D"], N) == 0
        assert xk.dgemm_async("N", "N", N, N, N, 1.0, m["D"], N, m["C"], N, 0.0, m["E"], N) == 0
        xk.memory_coherent_sync(N, N, m["E"], N)
        xk.memory_coherent_sync(N, N, m["D"], N)
    elif args.case == "dod":
        for name in ("A", "B", "C"):
            xk.memory_prefetch_async(N, N, m[name], N)
        xk.sync()
        xk.reset_stats()
        assert xk.dgemm_async("N", "N", N, N, N, 1.0, m["A"], N, m["B"], N, -1.0, m["C"], N) == 0
        xk.sync()
        xk.memory_coherent_sync(N, N, m["C"], N)
    elif args.case == "distribute":
        # the paper's data-on-device: 2D block-cyclic on a (1, world) grid,
        # transposed to the library's (world, 1) owner grid: every task reads peer tiles
        for name in ("A", "B", "C"):
            xk.distribute_2dbc_async(N, N, m[name], N, 1, args.world)
        xk.sync()
        out["dist_h2d"] = xk.get_stats()["h2d_bytes"][r]
        xk.reset_stats()
        assert xk.dgemm_async("N", "N", N, N, N, 1.0, m["A"], N, m["B"], N, -1.0, m["C"], N) == 0
        xk.sync()
        xk.memory_coherent_sync(N, N, m["C"], N)
    elif args.case == "big":
        # bench.py's launch configuration (alpha, beta, tile) on exact-integer inputs
        assert xk.dgemm("N", "N", N, N, N, 1.5, m["A"], N, m["B"], N, -0.75, m["C"], N) == 0
    elif args.case == "blas3":
        k = N // 2 + 3
        assert xk.dsyrk("L", "N", N, k, 2.0, m["A"], N, -1.0, m["C"], N) == 0
        snap = np.array(m["C"], order="F") if r == 0 else None
        assert xk.dsyr2k("U", "N", N, k, 1.0, m["A"], N, m["B"], N, 0.5, m["S"], N) == 0
        assert xk.dtrmm("L", "L", "N", "N", N, N, 1.0, m["S"], N, m["X"], N) == 0
        assert xk.dtrsm("L", "L", "N", "N", N, N, 1.5, m["L"], N, m["C"], N) == 0
    st = xk.get_stats()
    out["stats"] = {f: st[f][r] for f in ("h2d_bytes", "d2h_bytes", "p2p_in_bytes", "p2p_out_bytes", "tasks")}
    out["stats"]["forwards"] = st["forwards_inflight"] + st["forwards_valid"]
    out["topology"] = xk.get_topology()
    xk.finalize()

    if r == 0:
        import oracle
        c = C0
        if args.case == "gemm":
            ref = c["C"].copy(order="F")
            oracle.dgemm("N", "N", N, N, N, -2.0, c["A"], c["B"], 0.5, ref)
            check("C bitwise", np.array_equal(np.asarray(m["C"]), ref))
            refE = np.zeros((N, N), order="F")
            oracle.dgemm("T", "N", N, N, N, 1.0, c["A"], ref, 0.0, refE)
            check("E bitwise", np.array_equal(np.asarray(m["E"]), refE))
        elif args.case in ("dod", "distribute"):
            ref = c["C"].copy(order="F")
            oracle.dgemm("N", "N", N, N, N, 1.0, c["A"], c["B"], -1.0, ref)
            check("C bitwise", np.array_equal(np.asarray(m["C"]), ref))
        elif args.case == "big":
            # Freivalds, exact in FP64 (every partial sum is a multiple of 1/4 below 2^51)
            rng = np.random.default_rng(5)
            A_, B_, C_ = np.asarray(m["A"]), np.asarray(m["B"]), np.asarray(m["C"])
            for _ in range(2):
                x = rng.integers(-4, 5, N).astype(np.float64)
                check("freivalds", np.array_equal(C_ @ x, 1.5 * (A_ @ (B_ @ x)) - 0.75 * (c["C"] @ x)))
        elif args.case == "compose":
            refD = np.zeros((N, N), order="F")
            oracle.dgemm("N", "N", N, N, N, 1.0, c["A"], c["B"], 0.0, refD)
            refE = np.zeros((N, N), order="F")
            oracle.dgemm("N", "N", N, N, N, 1.0, refD, c["C"], 0.0, refE)
            check("D bitwise", np.array_equal(np.asarray(m["D"]), refD))
            check("E bitwise", np.array_equal(np.asarray(m["E"]), refE))
        elif args.case == "blas3":
            k = N // 2 + 3
            ref = c["C"].copy(order="F")
            oracle.dsyrk("L", "N", N, k, 2.0, c["A"], -1.0, ref)
            check("syrk bitwise (lower computed, upper untouched)", np.array_equal(snap, ref))
            ref2 = c["S"].copy(order="F")
            oracle.dsyr2k("U", "N", N, k, 1.0, c["A"], c["B"], 0.5, ref2)
            check("syr2k bitwise", np.array_equal(np.asarray(m["S"]), ref2))
            ref3 = c["X"].copy(order="F")
            oracle.dtrmm("L", "L", "N", "N", N, N, 1.0, ref2, ref3)
            check("trmm bitwise", np.array_equal(np.asarray(m["X"]), ref3))
            ref4 = ref.copy(order="F")
            oracle.dtrsm("L", "L", "N", "N", N, N, 1.5, c["L"], ref4)
            got = np.asarray(m["C"])
            Lt = np.tril(c["L"])
            resid = np.abs(Lt @ got - 1.5 * ref)
            bound = 4 * N * EPS * (np.abs(Lt) @ np.abs(got) + 1.5 * np.abs(ref))
            check("trsm residual", bool(np.all(resid <= bound)))
            check("trsm frobenius", bool(np.linalg.norm(got - ref4) <= 1e-13 * np.linalg.norm(ref4)))
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
