"""Pins for the CFD oracle (Fig. 15; Rodinia euler3d).

Independent anchors: the free-stream fixed point (bit-identical), finite stencil support
of the RK sweeps (exact), a float64 numpy re-derivation of one outer iteration written
here from the euler3d equations, closed-form task counts and the latch trace.
"""
import numpy as np
import pytest

from paper_conf_micro_zhengozsyc17_b200 import inputs

GAMMA, SMOOTH = 1.4, 0.2


def numpy_outer_iteration(sc):
    """One Copy / StepFactor / 3 x (Flux, TimeStep) outer iteration in float64."""
    G, n = sc.G, sc.G * sc.G
    U = sc.vars0.astype(np.float64).copy()
    ff = sc.ff.astype(np.float64)

    def prim(V):
        d, m, e = V[0], V[1:4], V[4]
        v = m / d
        sq = (v * v).sum(0)
        p = (GAMMA - 1) * (e - 0.5 * d * sq)
        c = np.sqrt(GAMMA * p / d)
        fm = np.stack([v[a] * m + (np.eye(3)[a][:, None] * p) for a in range(3)])  # fm[a][b] = v_a m_b + d_ab p
        fe = v * (e + p)
        return m, sq, p, c, fm, fe

    old = U.copy()
    _, sq, _, c, _, _ = prim(U)
    sf = 0.5 / (np.sqrt(sc.area.astype(np.float64)) * (np.sqrt(sq) + c))
    ffv = np.broadcast_to(ff[:, None], (5, n))
    for j in range(3):
        m, sq, p, c, fm, fe = prim(U)
        mf, sqf, pf, cf, fmf, fef = prim(ffv)
        flux = np.zeros((5, n))
        for face in range(4):
            nbr = sc.nb[face]
            nrm = sc.normals[face].astype(np.float64)
            nlen = np.sqrt((nrm * nrm).sum(0))
            inside = nbr >= 0
            k = np.where(inside, nbr, 0)
            Un = np.where(inside, U[:, k], ffv)
            mn, sqn, pn, cn, fmn, fen = prim(Un)
            visc = -nlen * SMOOTH * 0.5 * (np.sqrt(sq) + np.sqrt(sqn) + c + cn)
            flux += np.where(inside, visc * (U - Un), 0.0)
            # central: density uses momentum, energy uses fe, momentum b uses fm[a][b] (symmetric)
            cen = np.zeros((5, n))
            for a in range(3):
                fac = 0.5 * nrm[a]
                cen[0] += fac * (mn[a] + m[a])
                cen[4] += fac * (fen[a] + fe[a])
                for b in range(3):
                    cen[1 + b] += fac * (fmn[b][a] + fm[b][a])
            flux += cen
        U = old + (sf / (3 + 1 - j)) * flux
    return U


def test_far_field_state():
    ff = inputs.cfd_far_field().astype(np.float64)
    p = (GAMMA - 1) * (ff[4] - 0.5 * ff[1] ** 2 / ff[0])
    c = np.sqrt(GAMMA * p / ff[0])
    assert p == pytest.approx(1.0, rel=1e-6) and (ff[1] / ff[0]) / c == pytest.approx(1.2, rel=1e-6)


def test_free_stream_is_a_fixed_point(orc):
    sc = inputs.cfd_scene(G=32, n_outer=3, uniform=True)
    for fn in (orc.cfd_definition, orc.cfd_pipeline):
        r = fn(sc)
        assert np.array_equal(r["vars"], sc.vars0)


def test_stencil_support(orc):
    """After k RK steps every cell at Manhattan distance > k of a single perturbed cell
    is bit-identical to the free stream."""
    G = 32
    sc = inputs.cfd_scene(G=G, n_outer=2, uniform=True)
    r0, c0 = 11, 20
    sc.vars0[:, r0 * G + c0] *= np.float32(1.01)
    r = orc.cfd_pipeline(sc)
    k = 3 * sc.n_outer
    rr, cc = np.divmod(np.arange(G * G), G)
    far = np.abs(rr - r0) + np.abs(cc - c0) > k
    ff = sc.ff[:, None] * np.ones((1, G * G), np.float32)
    assert np.array_equal(r["vars"][:, far], ff[:, far])
    assert not np.array_equal(r["vars"][:, ~far], ff[:, ~far])   # and the perturbation did spread


def test_matches_float64_rederivation(orc):
    sc = inputs.cfd_scene(G=16, n_outer=1, bump_amp=0.3)
    r = orc.cfd_definition(sc)
    ref = numpy_outer_iteration(sc)
    assert np.allclose(r["vars"], ref, rtol=2e-5, atol=2e-5)


@pytest.mark.parametrize("G,n_outer", [(64, 2), (256, 1), (64, 10)])
def test_definition_equals_pipeline_and_counts(orc, G, n_outer):
    sc = inputs.cfd_scene(G=G, n_outer=n_outer)
    a = orc.cfd_definition(sc)
    b = orc.cfd_pipeline(sc, trace_cap=1 << 20)
    assert np.array_equal(a["vars"], b["vars"])
    tiles = G * G // sc.T
    assert b["n_copy"] == b["n_step"] == tiles * n_outer
    assert b["n_flux"] == b["n_time"] == 3 * tiles * n_outer
    tr = b["trace"]
    for st, k in enumerate(("n_copy", "n_step", "n_flux", "n_time")):
        ids = tr["id"][tr["stage"] == st]
        assert ids.size == b[k] and np.unique(ids).size == ids.size   # each (stage, tile, k) once
