"""CPU pins of the LDPC oracle (oracle/ldpc.c; Fig. 17, L59; DESIGN.md readings
R-L1..R-L6): single-parity-check codes against brute-force max-log decoding, exact channel
symmetry over a nonzero codeword of H, the noiseless closed-form message recursion, the
code construction, and definition == pipeline with the closed-form stage counts."""
import itertools

import numpy as np
import pytest

import oracle
from paper_conf_micro_zhengozsyc17_b200 import inputs


def scene_from(cv, N, dv, dc, llr, n_iter, alpha):
    ve = inputs.ldpc_var_edges(np.asarray(cv, np.int32), N, dv)
    return inputs.LdpcScene(N=N, M=N * dv // dc, dv=dv, dc=dc, check_vars=np.asarray(cv, np.int32), var_edges=ve,
                            llr=np.asarray(llr, np.float32), n_iter=n_iter, alpha=alpha)


def test_h_is_regular_without_repeated_variables():
    sc = inputs.ldpc_scene(n_frames=1)
    rows = sc.check_vars.reshape(sc.M, sc.dc)
    assert all(len(set(r)) == sc.dc for r in rows.tolist())
    assert np.all(np.bincount(sc.check_vars, minlength=sc.N) == sc.dv)
    assert sc.M == 1024 and sc.N == 2048


@pytest.mark.parametrize("dc", [2, 3, 6])
def test_single_parity_checks_equal_brute_force_max_log(dc):
    """dv = 1: H is a set of disjoint single parity checks (a cycle-free Tanner graph), so
    min-sum with alpha = 1 is exact max-log decoding: P_n = max over even-weight words with
    c_n = 0 of sum x_k L_k / 2 minus the same with c_n = 1, times 2 (x = 1 - 2c)."""
    rng = np.random.default_rng(dc)
    M = 40
    N = M * dc
    llr = rng.normal(1.0, 2.0, size=(3, N)).astype(np.float32)
    cv = np.arange(N, dtype=np.int32)                      # check m holds variables m*dc..m*dc+dc-1
    sc = scene_from(cv, N, 1, dc, llr, n_iter=2, alpha=1.0)
    got = oracle.ldpc_definition(sc)["post"]
    words = [w for w in itertools.product((0, 1), repeat=dc) if sum(w) % 2 == 0]
    for f in range(3):
        for m in range(M):
            L = llr[f, m * dc:(m + 1) * dc].astype(np.float64)
            for n in range(dc):
                best = {0: -np.inf, 1: -np.inf}
                for w in words:
                    v = sum((1 - 2 * b) * L[k] for k, b in enumerate(w)) / 2.0
                    best[w[n]] = max(best[w[n]], v)
                assert got[f, m * dc + n] == pytest.approx(best[0] - best[1], rel=1e-6, abs=1e-6)


def gf2_nullspace_vector(H):
    """One nonzero codeword of H (rows = checks) by Gaussian elimination over GF(2)."""
    H = H.copy() % 2
    M, N = H.shape
    piv_cols, r = [], 0
    for c in range(N):
        rows = np.nonzero(H[r:, c])[0]
        if rows.size == 0:
            continue
        p = r + rows[0]
        H[[r, p]] = H[[p, r]]
        for i in range(M):
            if i != r and H[i, c]:
                H[i] ^= H[r]
        piv_cols.append(c)
        r += 1
        if r == M:
            break
    free = [c for c in range(N) if c not in set(piv_cols)]
    x = np.zeros(N, np.uint8)
    x[free[0]] = 1
    for i, c in enumerate(piv_cols):
        x[c] = H[i, free[0]]
    return x


def test_channel_symmetry_is_exact():
    """Transmitting codeword x' instead of 0 flips the signs of exactly the LLRs where x'=1;
    min-sum (signs multiply, magnitudes and sums only negate) must return bit-for-bit the
    negated posteriors there and identical error counts relative to x'."""
    sc = inputs.ldpc_scene(n_frames=3, N=512, n_iter=12)
    H = np.zeros((sc.M, sc.N), np.uint8)
    H[np.repeat(np.arange(sc.M), sc.dc), sc.check_vars] = 1
    x = gf2_nullspace_vector(H)
    assert x.any() and not (H.astype(np.int64) @ x % 2).any()
    flip = np.where(x == 1, -1.0, 1.0).astype(np.float32)
    a = oracle.ldpc_definition(sc)
    b = oracle.ldpc_definition(sc, llr=sc.llr * flip)
    assert np.array_equal(b["post"], a["post"] * flip)


def test_noiseless_closed_form_recursion():
    """All LLRs = 10: every message is positive and equal, so v_0 = 10, c_k = alpha v_k,
    v_{k+1} = 10 + (dv - 1) c_k and P_k = 10 + dv c_k (exact binary fractions)."""
    sc = inputs.ldpc_scene(n_frames=1, N=256, n_iter=5)
    sc.llr[:] = 10.0
    for iters in range(1, 6):
        r = oracle.ldpc_definition(sc, n_iter=iters)
        v = 10.0
        for _ in range(iters):
            c = 0.75 * v
            P = 10.0 + 3 * c
            v = 10.0 + 2 * c
        assert np.all(r["post"] == np.float32(P)) and not r["errors"].any()


@pytest.mark.parametrize("N", [1024, 2048])
def test_pipeline_chunking_is_exact(N):
    """Chunked items with latches reproduce the per-frame definition for every chunking."""
    sc = inputs.ldpc_scene(n_frames=3, N=N, n_iter=6)
    a = oracle.ldpc_definition(sc)
    b = oracle.ldpc_pipeline(sc)
    assert np.array_equal(a["post"], b["post"]) and np.array_equal(a["errors"], b["errors"])
    assert b["deq"] == [3, 3 * 6 * sc.nc_chk, 3 * 6 * sc.nc_var, 3 * 6 * sc.nc_var]


def test_definition_equals_pipeline_and_counts():
    sc = inputs.ldpc_scene(n_frames=5, N=1024, n_iter=15)
    a = oracle.ldpc_definition(sc)
    b = oracle.ldpc_pipeline(sc)
    assert np.array_equal(a["post"], b["post"]) and np.array_equal(a["errors"], b["errors"])
    # items (reading R-L6): Initialize per frame, then per iteration nc_chk C2V chunks and
    # nc_var V2C + nc_var ProbVar chunks (chunks of <= 256 checks / variables)
    assert (sc.nc_chk, sc.nc_var) == (2, 4)
    assert b["deq"] == [5, 5 * 15 * 2, 5 * 15 * 4, 5 * 15 * 4]
    # the decoder converges on this channel (errors reach 0 for every frame)
    assert not a["errors"][:, -1].any() and a["errors"][:, 0].sum() > 0
