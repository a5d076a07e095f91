"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Bar: bitwise for fields and
the dt history (both sides are IEEE fp64 with no contraction, reading A8);
north_star tolerances as the fallback gate: field_summary totals 1e-10
relative, per-cell 1e-9 (A14 metric).
"""
from __future__ import annotations

import numpy as np
import pytest

from oracle import Oracle
from workloads import (bm_deck, colliding_slab_deck, contact_deck, fuzz_deck, point_deck, quiescent_deck,
                       random_state_fields, symmetric_deck)

pytestmark = pytest.mark.gpu

STATE = ("density0", "energy0", "xvel0", "yvel0")
SUMMARY_TOL = 1e-10
CELL_TOL = 1e-9


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def make_gpu(deck, **kw):
    from paper_conf_cluster_regulymg15_b200 import Clover
    return Clover(deck, **kw)


def rel_cell(a, b):
    """A14: abs(a-b) <= tol*max(|a|,|b|,s_f), s_f = 1e-12*max|f|."""
    s = 1e-12 * max(np.abs(a).max(), np.abs(b).max(), 1e-300)
    den = np.maximum(np.maximum(np.abs(a), np.abs(b)), s)
    return float((np.abs(a - b) / den).max())


def assert_fields_equal(gpu, ora, names=STATE, bitwise=True, ctx=""):
    for f in names:
        a, b = gpu.read(f), ora.read(f)
        assert a.shape == b.shape
        if bitwise:
            if not np.array_equal(a, b):
                bad = np.argwhere(a != b)
                k, j = bad[0]
                raise AssertionError(f"{ctx} {f}: {len(bad)} differ, first (k={k + 1}, j={j + 1}) "
                                     f"gpu={a[k, j]!r} oracle={b[k, j]!r} rel={rel_cell(a, b):.3e}")
        assert rel_cell(a, b) <= CELL_TOL, (ctx, f)


def assert_summary_close(gs, os_):
    for key in ("vol", "mass", "ie", "ke", "press"):
        a, b = gs[key], os_[key]
        if b == 0.0:
            assert a == 0.0, key
        else:
            assert abs(a - b) / abs(b) <= SUMMARY_TOL, (key, a, b)


def test_init_matches_oracle(torch_cuda):
    for deck in (bm_deck(64), fuzz_deck(1), fuzz_deck(4)):
        g, o = make_gpu(deck), Oracle(deck)
        assert_fields_equal(g, o)
        assert_summary_close(g.field_summary(), o.field_summary())
        for f in ("pressure", "soundspeed"):
            assert np.array_equal(g.read(f), o.read(f)), f


def test_stage_parity_bm64(torch_cuda):
    """Kernel-by-kernel parity on step 1 and 2 of bm64 (x-first then y-first)."""
    deck = bm_deck(64)
    deck["max_timestep"] = 1.0
    for step in range(2):
        g, o = make_gpu(deck), Oracle(deck)
        if step:
            g.step(1); o.step(1)
        g.debug_partial_step(1)
        o.run_stage("timestep")
        assert np.array_equal(g.debug_read("q", "cell"), o.read("viscosity"))
        g2 = make_gpu(deck)
        if step:
            g2.step(1)
        g2.debug_partial_step(3)
        o.run_stage("pdv_predict"); o.run_stage("accelerate"); o.run_stage("pdv_correct")
        o.run_stage("flux_calc")
        for buf, kind, name in (("d1", "cell", "density1"), ("e1", "cell", "energy1"),
                                ("u1", "xvel", "xvel1"), ("v1", "yvel", "yvel1"),
                                ("fx", "xface", "vol_flux_x"), ("fy", "yface", "vol_flux_y")):
            a, b = g2.debug_read(buf, kind), o.read(name)
            assert np.array_equal(a, b), (step, name, rel_cell(a, b))
        g3 = make_gpu(deck)
        g3.debug_set_fusion(False)  # the separate advec_cell kernel (mass flux kept)
        if step:
            g3.step(1)
        g3.debug_partial_step(4)
        o.run_stage("adv_cell1")
        mname = "mass_flux_x" if step == 0 else "mass_flux_y"
        mkind = "xface" if step == 0 else "yface"
        mbuf = "mx" if step == 0 else "my"
        for buf, kind, name in (("d2", "cell", "density1"), ("e2", "cell", "energy1"),
                                (mbuf, mkind, mname)):
            a, b = g3.debug_read(buf, kind), o.read(name)
            assert np.array_equal(a, b), (step, name, rel_cell(a, b))


def test_fused_x_sweep_stage_parity(torch_cuda):
    """The fused x sweep (advec_cell x + advec_mom x in one kernel) against
    the oracle's adv_cell1 + adv_mom1 stages, step 1 (x first)."""
    for deck in (bm_deck(64), fuzz_deck(3)):
        deck["max_timestep"] = 1.0
        g, o = make_gpu(deck), Oracle(deck)
        g.debug_partial_step(5)
        for st in ("timestep", "pdv_predict", "accelerate", "pdv_correct", "flux_calc",
                   "adv_cell1", "adv_mom1"):
            o.run_stage(st)
        for buf, kind, name in (("d2", "cell", "density1"), ("e2", "cell", "energy1"),
                                ("u2", "xvel", "xvel1"), ("v2", "yvel", "yvel1")):
            a, b = g.debug_read(buf, kind), o.read(name)
            assert np.array_equal(a, b), (name, rel_cell(a, b))


def test_fused_y_sweep_stage_parity(torch_cuda):
    """The fused y sweep (wall bands + advec_cell y + advec_mom y in one
    kernel) against the oracle's adv_cell1 + adv_mom1 stages of step 2
    (y first), single chunk and 2x1 chunks (x chunk boundary: halo columns
    recomputed)."""
    for deck, kw in ((bm_deck(64), {}), (fuzz_deck(3), {}), (fuzz_deck(5), dict(px=2, py=1))):
        deck["max_timestep"] = 1.0
        g, o = make_gpu(deck, **kw), Oracle(deck)
        g.step(1)
        o.step(1)
        g.debug_partial_step(5)
        for st in ("timestep", "pdv_predict", "accelerate", "pdv_correct", "flux_calc",
                   "adv_cell1", "adv_mom1"):
            o.run_stage(st)
        for buf, kind, name in (("d2", "cell", "density1"), ("e2", "cell", "energy1"),
                                ("u2", "xvel", "xvel1"), ("v2", "yvel", "yvel1")):
            a, b = g.debug_read(buf, kind), o.read(name)
            assert np.array_equal(a, b), (name, rel_cell(a, b))


@pytest.mark.parametrize("case", ["bm", "fuzz", "random", "tiny", "ragged", "chunks_1x3",
                                  "chunks_3x1"])
def test_fused_and_separate_x_sweep_identical(torch_cuda, case):
    """Fused and separate x and y sweeps give bit-identical states (halo
    included: the next kernels read the mirrors/exchanged halos both paths
    produce)."""
    kw = {}
    fields = None
    if case == "bm":
        deck = bm_deck(96, 80)
    elif case == "fuzz":
        deck = fuzz_deck(7)
    elif case == "ragged":
        deck = bm_deck(61, 37)
    elif case == "chunks_1x3":
        deck = fuzz_deck(11)
        kw = dict(px=1, py=3)
    elif case == "chunks_3x1":  # fused y with x chunk boundaries
        deck = fuzz_deck(12)
        kw = dict(px=3, py=1)
    else:
        deck = bm_deck(70, 50)
        deck["max_timestep"] = 1.0
        fields = random_state_fields(13, 70, 50)
        if case == "tiny":
            for f in ("xvel0", "yvel0"):
                fields[f][:, :30] *= 1e-303
    runs = []
    for fused in (True, False):
        g = make_gpu(deck, **kw)
        g.debug_set_fusion(fused)
        if fields is not None:
            g.load_state(fields)
        g.step(6)
        runs.append(g)
    assert np.array_equal(runs[0].dt_history(1, 6), runs[1].dt_history(1, 6))
    for f in STATE:
        a, b = runs[0].read(f), runs[1].read(f)
        assert np.array_equal(a, b) and np.array_equal(np.signbit(a), np.signbit(b)), (case, f)


def test_bm64_20_steps_bitwise(torch_cuda):
    deck = bm_deck(64, end_step=20)
    g, o = make_gpu(deck), Oracle(deck)
    g.step(20)
    dts = o.step(20)
    assert np.array_equal(g.dt_history(1, 20), dts)
    assert_fields_equal(g, o, ctx="bm64")
    assert_summary_close(g.field_summary(), o.field_summary())
    c = g.clock()
    assert c["step"] == 20 and c["time"] == o.clock()["time"]


@pytest.mark.parametrize("mirror", [0, 1])
@pytest.mark.parametrize("seed", [0, 1, 2, 3, 4, 5])
def test_fuzz_decks_bitwise(torch_cuda, seed, mirror):
    deck = fuzz_deck(seed)
    deck["face_mirror"] = mirror
    g, o = make_gpu(deck), Oracle(deck)
    g.step(10)
    dts = o.step(10)
    assert np.array_equal(g.dt_history(1, 10), dts)
    assert_fields_equal(g, o, ctx=f"fuzz{seed}/m{mirror}")
    assert_summary_close(g.field_summary(), o.field_summary())


@pytest.mark.parametrize("shape", [(4, 4), (5, 7), (33, 9), (65, 47), (31, 40), (96, 17)])
def test_ragged_meshes_bitwise(torch_cuda, shape):
    nx, ny = shape
    deck = fuzz_deck(11, nx=nx, ny=ny)
    g, o = make_gpu(deck), Oracle(deck)
    g.step(6)
    dts = o.step(6)
    assert np.array_equal(g.dt_history(1, 6), dts)
    assert_fields_equal(g, o, ctx=str(shape))


@pytest.mark.parametrize("case", [(64, 64, None, None, 1, 1), (72, 56, 30, 21, 1, 1),
                                  (96, 80, None, None, 2, 2)])
def test_point_and_circle_decks_bitwise(torch_cuda, case):
    """Point and circle state shapes: a point blast next to
    a resting and a moving circle, on a dyadic and a ragged mesh and on 2x2
    local chunks; fields, dt history and summary against the oracle."""
    nx, ny, jp, kp, px, py = case
    deck = point_deck(nx, ny, 25, jp=jp, kp=kp)
    g, o = make_gpu(deck, px=px, py=py), Oracle(deck)
    assert_fields_equal(g, o, ctx=f"point{case} init")
    g.step(25)
    dts = o.step(25)
    assert np.array_equal(g.dt_history(1, 25), dts)
    assert_fields_equal(g, o, ctx=f"point{case}")
    assert_summary_close(g.field_summary(), o.field_summary())


@pytest.mark.parametrize("smooth", [False, True])
def test_random_state_bitwise(torch_cuda, smooth):
    nx, ny = 70, 50
    deck = bm_deck(nx, ny)
    deck["max_timestep"] = 1.0
    fields = random_state_fields(5, nx, ny, smooth=smooth)
    g, o = make_gpu(deck), Oracle(deck)
    g.load_state(fields)
    o.load_state(fields)
    assert_fields_equal(g, o, ctx="loaded")
    g.step(4)
    dts = o.step(4)
    assert np.array_equal(g.dt_history(1, 4), dts)
    assert_fields_equal(g, o, ctx="random")
    assert np.array_equal(g.read("viscosity"), o.read("viscosity"))


@pytest.mark.parametrize("scale", [1e-300, 1e-306])
def test_tiny_numerators_take_the_ieee_fixup_bitwise(torch_cuda, scale):
    """Velocities of 1e-300 (and subnormal-adjacent 1e-306) in the left half:
    numerators below 2^-900 make DivFast flag, so those warp segments are
    recomputed by the IEEE fixup launches.  Bitwise vs the
    oracle, and the fixup path must actually have run."""
    nx, ny = 96, 64
    deck = bm_deck(nx, ny)
    deck["max_timestep"] = 1.0
    fields = random_state_fields(9, nx, ny)
    for f in ("xvel0", "yvel0"):
        fields[f][:, : (nx + 1) // 2] *= scale
    g, o = make_gpu(deck), Oracle(deck)
    g.load_state(fields)
    o.load_state(fields)
    g.step(3)
    dts = o.step(3)
    assert np.array_equal(g.dt_history(1, 3), dts)
    assert_fields_equal(g, o, ctx=f"tiny {scale}")
    assert np.array_equal(g.read("viscosity"), o.read("viscosity"))
    assert g.debug_fix_count() > 0


@pytest.mark.parametrize("axis", ["x", "y", "xy"])
@pytest.mark.parametrize("pxy", [(1, 1), (2, 2), (1, 3)])
def test_divergence_limit_decks_bitwise(torch_cuda, axis, pxy):
    """calc_dt's divergence term (c.4 dtdivt) decides dt on steps 1-2 of the
    colliding-slab decks (oracle pin test_p2c_*): the kernel's min-w path
    must give the same dt history, fields and summary bit for bit, on one
    chunk and across chunk boundaries (the collision column sits on the
    x = 5 chunk edge of the 2x2 layout)."""
    n = 72
    deck = colliding_slab_deck(n, axis, 1.0, end_step=12)
    g, o = make_gpu(deck, px=pxy[0], py=pxy[1]), Oracle(deck)
    g.step(12)
    dts = o.step(12)
    factor = 0.175 if axis == "xy" else 0.35
    assert abs(dts[0] / (factor * 10.0 / n) - 1.0) < 1e-15  # dtdivt binds (closed form)
    assert np.array_equal(g.dt_history(1, 12), dts)
    assert_fields_equal(g, o, ctx=f"slab {axis} {pxy}")
    assert_summary_close(g.field_summary(), o.field_summary())


@pytest.mark.parametrize("mirror", [0, 1])
def test_byte_equal_to_oracle_cli_dump(torch_cuda, tmp_path, mirror):
    """the oracle's command-line driver (text deck in,
    raw fp64 dumps out) and clover_read_field share one layout, so parity is
    a byte compare of the files: state, EOS fields, viscosity and the volume
    fluxes (the fused sweeps never store the mass fluxes)."""
    import subprocess

    import oracle
    from oracle.deck import deck_to_text
    deck = fuzz_deck(6, nx=45, ny=38)
    deck["face_mirror"] = mirror
    oracle.build()
    (tmp_path / "clover.in").write_text(deck_to_text(deck))
    r = subprocess.run([oracle.CLI_PATH, "--steps", "8", "--dump", str(tmp_path),
                        str(tmp_path / "clover.in")], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    g = make_gpu(deck)
    g.step(8)
    for f in ("density0", "energy0", "pressure", "soundspeed", "viscosity", "xvel0", "yvel0",
              "vol_flux_x", "vol_flux_y"):
        assert g.read(f).astype("<f8").tobytes() == (tmp_path / f"{f}.f64").read_bytes(), f


def test_invariant_decks(torch_cuda):
    for deck in (quiescent_deck(64), contact_deck(64), symmetric_deck(64)):
        g, o = make_gpu(deck), Oracle(deck)
        g.step(20)
        o.step(20)
        assert_fields_equal(g, o)


@pytest.mark.parametrize("pxy", [(2, 1), (1, 2), (2, 2), (3, 2), (1, 4)])
def test_local_chunk_decomposition_bitwise(torch_cuda, pxy):
    """px*py chunks on one GPU (device-to-device halo exchange) give the same
    bits as one chunk and as the oracle, including the summary."""
    deck = bm_deck(96, 80)
    deck["max_timestep"] = 1.0
    one = make_gpu(deck)
    many = make_gpu(deck, px=pxy[0], py=pxy[1])
    o = Oracle(deck)
    one.step(12)
    many.step(12)
    o.step(12)
    for f in STATE:
        assert np.array_equal(many.read(f), one.read(f)), f
    assert_fields_equal(many, o)
    assert many.field_summary() == one.field_summary()


@pytest.mark.parametrize("pxy", [(2, 1), (1, 2), (2, 2), (3, 2), (2, 4)])
def test_virtual_remote_exchange_bitwise(torch_cuda, pxy):
    """Every chunk boundary through the multi-GPU packing path (pack ->
    staging -> unpack, the NCCL pair replaced by a device copy): same bits
    as one chunk, including the dt history."""
    deck = fuzz_deck(9, nx=96, ny=80)
    one = make_gpu(deck)
    many = make_gpu(deck, px=pxy[0], py=pxy[1])
    many.debug_set_virtual_remote(True)
    one.step(10)
    many.step(10)
    for f in STATE:
        assert np.array_equal(many.read(f), one.read(f)), f
    assert np.array_equal(many.dt_history(1, 10), one.dt_history(1, 10))


@pytest.mark.parametrize("pxy", [(2, 2), (1, 3), (2, 4)])
def test_virtual_remote_through_nccl_bitwise(torch_cuda, pxy):
    """the multi-GPU exchange code with NCCL itself executing.
    A one-rank NCCL communicator carries every chunk-boundary message as an
    ncclSend/ncclRecv pair to self (paired exactly as two ranks' lists pair
    up) and dt through a one-rank ncclAllReduce(MIN), all captured in the
    step's CUDA graph: same bits as one chunk, dt history included."""
    deck = fuzz_deck(9, nx=96, ny=80)
    one = make_gpu(deck)
    many = make_gpu(deck, px=pxy[0], py=pxy[1])
    many.debug_set_virtual_remote(True, nccl=True)
    one.step(10)
    many.step(10)
    for f in STATE:
        assert np.array_equal(many.read(f), one.read(f)), f
    assert np.array_equal(many.dt_history(1, 10), one.dt_history(1, 10))
    assert many.field_summary() == one.field_summary()


@pytest.mark.parametrize("nccl", [False, True])
@pytest.mark.parametrize("py", [2, 3, 5])
def test_boundary_first_overlap_bitwise(torch_cuda, nccl, py):
    """S:8(e) boundary-strip-first + interior overlap: with y strips whose
    exchanges take the remote path, each fused kernel runs the segments next
    to a chunk boundary first, then the exchange (device copy or one-rank
    NCCL) on a second stream while the interior segments run.  Same bits as
    without the overlap and as one chunk (fields, dt history), both sweep
    orders, graphs on; more launches per step than without."""
    deck = fuzz_deck(16, nx=64, ny=40 * py)
    deck["max_timestep"] = 1.0
    one = make_gpu(deck)
    ov = make_gpu(deck, px=1, py=py)
    ov.debug_set_virtual_remote(True, nccl=nccl)
    ov.set_deep_halo(False)  # (overlap is for the per-phase exchange schedule)
    ov.debug_set_overlap(True)
    plain = make_gpu(deck, px=1, py=py)
    plain.debug_set_virtual_remote(True, nccl=nccl)
    plain.set_deep_halo(False)
    plain.debug_set_overlap(False)
    assert ov.kernels_per_step() > plain.kernels_per_step()
    for g in (one, ov, plain):
        g.step(9)
    for f in STATE:
        a = one.read(f)
        assert np.array_equal(ov.read(f), a), f
        assert np.array_equal(plain.read(f), a), f
    assert np.array_equal(ov.dt_history(1, 9), one.dt_history(1, 9))


@pytest.mark.parametrize("seed,pxy", [(8, (1, 2)), (9, (1, 4)), (10, (2, 3)), (11, (1, 5)),
                                      (12, (2, 1)), (13, (3, 1)), (14, (4, 2)), (15, (3, 3))])
def test_fused_sweeps_across_chunk_boundaries(torch_cuda, seed, pxy):
    """at chunk boundaries the fused
    sweeps recompute the neighbour's first post-sweep rows (y) / columns (x)
    from depth-4 input halos.  Same bits as the separate cell / momentum
    kernels with their extra exchanges (fusion walls_only) and as one chunk,
    on fuzz decks (flow across the boundaries) for 12 steps (both sweep
    orders), local and virtual-remote exchange."""
    deck = fuzz_deck(seed, nx=72, ny=96)
    deck["max_timestep"] = 1.0
    one = make_gpu(deck)
    fused = make_gpu(deck, px=pxy[0], py=pxy[1])
    split = make_gpu(deck, px=pxy[0], py=pxy[1])
    split.debug_set_fusion(True, walls_only=True)
    remote = make_gpu(deck, px=pxy[0], py=pxy[1])
    remote.debug_set_virtual_remote(True)
    assert fused.kernels_per_step() < split.kernels_per_step()
    for g in (one, fused, split, remote):
        g.step(12)
    for f in STATE:
        a = one.read(f)
        for g in (fused, split, remote):
            assert np.array_equal(g.read(f), a), f
    assert np.array_equal(fused.dt_history(1, 12), one.dt_history(1, 12))


@pytest.mark.parametrize("seed,py,mode", [(8, 2, "local"), (9, 3, "local"), (10, 5, "local"),
                                           (11, 2, "remote"), (12, 4, "remote"), (13, 3, "nccl"),
                                           (14, 6, "nccl")])
def test_deep_halo_bitwise(torch_cuda, seed, py, mode):
    """S:8(f) f1 deep halos: one 7-row state exchange per step, every kernel
    run over the rows of its y neighbours it would otherwise receive.  Fuzz
    decks (flow across the boundaries), 12 steps (both sweep orders): fields,
    dt history and summary bitwise equal to one chunk and to the per-phase
    exchange schedule; local chunks, virtual remote (device copy) and NCCL
    messages."""
    deck = fuzz_deck(seed, nx=72, ny=112)
    deck["max_timestep"] = 1.0
    one = make_gpu(deck)
    deep = make_gpu(deck, px=1, py=py)
    plain = make_gpu(deck, px=1, py=py)
    if mode != "local":
        for g in (deep, plain):
            g.debug_set_virtual_remote(True, nccl=(mode == "nccl"))
    deep.set_deep_halo(True)
    plain.set_deep_halo(False)
    assert deep.deep_halo_active() and not plain.deep_halo_active()
    for g in (one, deep, plain):
        g.step(12)
    for f in STATE:
        a = one.read(f)
        assert np.array_equal(deep.read(f), a), f
        assert np.array_equal(plain.read(f), a), f
    assert np.array_equal(deep.dt_history(1, 12), one.dt_history(1, 12))
    assert deep.field_summary() == one.field_summary()


@pytest.mark.parametrize("py,deep", [(2, True), (3, True), (6, True), (3, False)])
def test_lsa_device_initiated_halo_stores_bitwise(torch_cuda, py, deep):
    """S:8(f) f1 device-initiated halo stores: every halo message is packed
    straight into its receiver's slot of an NCCL symmetric window (one-rank
    communicator, peer mapping from the window), LSA barriers around the
    unpack; with deep halos (one 7-row state exchange per step) and the
    per-phase schedule.  Fuzz decks, 12 steps: fields, dt history and summary
    bitwise equal to one chunk."""
    deck = fuzz_deck(17 + py, nx=72, ny=112)
    deck["max_timestep"] = 1.0
    one = make_gpu(deck)
    g = make_gpu(deck, px=1, py=py)
    g.debug_set_virtual_remote(True, lsa=True)
    g.set_deep_halo(deep)
    assert g.deep_halo_active() == deep
    one.step(12)
    g.step(7)
    g.set_graphs(False)  # direct launches: the same exchange sequence outside a graph
    g.step(5)
    for f in STATE:
        assert np.array_equal(g.read(f), one.read(f)), f
    assert np.array_equal(g.dt_history(1, 12), one.dt_history(1, 12))
    assert g.field_summary() == one.field_summary()


@pytest.mark.parametrize("pxy", [(2, 2), (3, 2)])
def test_lsa_halo_stores_2d_layouts(torch_cuda, pxy):
    """Device-initiated stores on 2D chunk grids (x and y messages, the
    4-chunk corners through the second axis): bitwise equal to one chunk."""
    deck = fuzz_deck(23, nx=96, ny=80)
    deck["max_timestep"] = 1.0
    one, g = make_gpu(deck), make_gpu(deck, px=pxy[0], py=pxy[1])
    g.debug_set_virtual_remote(True, lsa=True)
    one.step(10)
    g.step(10)
    for f in STATE:
        assert np.array_equal(g.read(f), one.read(f)), f
    assert np.array_equal(g.dt_history(1, 10), one.dt_history(1, 10))


@pytest.mark.parametrize("pxy,deep", [((1, 4), True), ((1, 4), False), ((2, 3), False),
                                      ((1, 16), False)])
def test_batched_chunk_launches_bitwise(torch_cuda, monkeypatch, pxy, deep):
    """Several chunks in one process: every streaming kernel and its fixup is
    one launch for all chunks (blockIdx.z = chunk, KBatch) -- the same bits
    as one launch per chunk (CLOVER_BATCH=0) and as one chunk."""
    deck = fuzz_deck(31, nx=80, ny=128)
    deck["max_timestep"] = 1.0
    one = make_gpu(deck)
    b = make_gpu(deck, px=pxy[0], py=pxy[1])
    monkeypatch.setenv("CLOVER_BATCH", "0")
    per = make_gpu(deck, px=pxy[0], py=pxy[1])
    for g in (b, per):
        g.set_deep_halo(deep)
    for g in (one, b, per):
        g.step(11)
    for f in STATE:
        a = one.read(f)
        assert np.array_equal(b.read(f), a), f
        assert np.array_equal(per.read(f), a), f
    assert np.array_equal(b.dt_history(1, 11), one.dt_history(1, 11))


@pytest.mark.parametrize("pxy", [(1, 1), (1, 2)])
def test_segment_chains_on_off_bitwise(torch_cuda, monkeypatch, pxy):
    """Segment chains (seg_chain: the launch order walks consecutive row
    segments in consecutive waves) change only which block runs which rows
    when: a mesh large enough for several waves and chains on every kernel
    (3840 x 4096; 1 x 2 batched chunks of 3840 x 2048 with deep halos) gives
    the same bits with chains on and off (CLOVER_CHAIN=0).  The bm 3840^2
    oracle comparison (test_full_size_first_steps) runs with chains on."""
    deck = fuzz_deck(5, nx=3840, ny=4096)
    deck["max_timestep"] = 1.0
    on = make_gpu(deck, px=pxy[0], py=pxy[1])
    monkeypatch.setenv("CLOVER_CHAIN", "0")
    off = make_gpu(deck, px=pxy[0], py=pxy[1])
    for g in (on, off):
        g.step(4)
    for f in STATE:
        assert np.array_equal(on.read(f), off.read(f)), f
    assert np.array_equal(on.dt_history(1, 4), off.dt_history(1, 4))


def test_deep_halo_bm_blast_and_toggles(torch_cuda):
    """The bm blast crossing 1x4 strip boundaries for 40 steps with deep
    halos switched on and off between steps (the state halo is refreshed 7
    deep when a deep step follows a plain one), graphs on and off: bitwise
    equal to one chunk and to the oracle."""
    deck = bm_deck(128, end_step=40)
    one, g = make_gpu(deck), make_gpu(deck, px=1, py=4)
    g.set_deep_halo(True)
    assert g.deep_halo_active()
    g.step(10)
    g.set_deep_halo(False)
    g.step(5)
    g.set_deep_halo(True)
    g.set_graphs(False)
    g.step(10)
    g.set_graphs(True)
    g.step(15)
    one.step(40)
    for f in STATE:
        assert np.array_equal(g.read(f), one.read(f)), f
    assert np.array_equal(g.dt_history(1, 40), one.dt_history(1, 40))
    o = Oracle(deck)
    o.step(40)
    assert_fields_equal(g, o, ctx="deep bm 1x4")


@pytest.mark.parametrize("pxy,ny", [((2, 2), 112), ((1, 8), 112), ((1, 1), 112)])
def test_deep_halo_inactive_layouts(torch_cuda, pxy, ny):
    """Deep halos need y strips (px == 1, py > 1) of at least 16 rows; other
    layouts keep the per-phase schedule (the setting has no effect) and stay
    bitwise."""
    deck = fuzz_deck(15, nx=72, ny=ny)
    deck["max_timestep"] = 1.0
    one, g = make_gpu(deck), make_gpu(deck, px=pxy[0], py=pxy[1])
    g.set_deep_halo(True)
    assert not g.deep_halo_active()
    one.step(6)
    g.step(6)
    for f in STATE:
        assert np.array_equal(g.read(f), one.read(f)), f


@pytest.mark.parametrize("seed,pxy", [(8, (2, 3)), (9, (3, 2)), (9, (2, 4)), (12, (4, 4)),
                                      (13, (3, 3))])
def test_local_chunks_fuzz(torch_cuda, seed, pxy):
    """Fuzz decks put flow on the 4-chunk corners (the bm deck never does):
    the corner halos of node/face fields must be refreshed by the second
    exchange axis (regression: x-face Mx(nx+3, ny+1) was once missed)."""
    deck = fuzz_deck(seed, nx=96, ny=80)
    deck["max_timestep"] = 1.0
    one, many = make_gpu(deck), make_gpu(deck, px=pxy[0], py=pxy[1])
    one.step(12)
    many.step(12)
    for f in STATE:
        assert np.array_equal(many.read(f), one.read(f)), f
    assert np.array_equal(many.dt_history(1, 12), one.dt_history(1, 12))


def test_graphs_on_off_identical(torch_cuda):
    deck = fuzz_deck(2)
    a, b = make_gpu(deck), make_gpu(deck)
    b.set_graphs(False)
    a.step(7)
    b.step(7)
    for f in STATE:
        assert np.array_equal(a.read(f), b.read(f))


def test_step_host_matches_device_path(torch_cuda):
    nx = ny = 48
    deck = bm_deck(nx, ny)
    f = random_state_fields(3, nx, ny, smooth=True)
    a = make_gpu(deck)
    outs = {k: np.empty_like(v) for k, v in f.items()}
    a.step_host(3, f, outs)
    o = Oracle(deck)
    o.load_state(f)
    o.step(3)
    for k in STATE:
        assert np.array_equal(outs[k], o.read(k)), k


@pytest.mark.parametrize("pxy", [(1, 3), (2, 2)])
def test_step_host_on_several_chunks(torch_cuda, pxy):
    """clover_step_host on a multi-chunk context: every chunk takes its block
    of the global host arrays in and out; same bits as one chunk."""
    nx, ny = 64, 96
    deck = bm_deck(nx, ny)
    f = random_state_fields(5, nx, ny, smooth=True)
    one, many = make_gpu(deck), make_gpu(deck, px=pxy[0], py=pxy[1])
    o1 = {k: np.empty_like(v) for k, v in f.items()}
    om = {k: np.full_like(v, np.nan) for k, v in f.items()}
    one.step_host(4, f, o1)
    many.step_host(4, f, om)
    for k in STATE:
        assert np.array_equal(om[k], o1[k]), k


def test_small_dt_error_is_latched(torch_cuda):
    from paper_conf_cluster_regulymg15_b200 import CloverError
    deck = bm_deck(32)
    deck["dtmin"] = 0.5  # every dt is smaller than this
    g = make_gpu(deck)
    g.step(1)
    with pytest.raises(CloverError) as ei:
        g.sync()
    assert ei.value.code == -5


def test_negative_volume_is_latched(torch_cuda):
    """SURVEY 8(b) CLOVER_ERR_NEG_VOLUME: with the CFL safety factors raised
    20x the step (dt = 1.85 on bm64) is far beyond stability: PdV's corrector
    turns cells inside out on step 1 already (the oracle's density1 after
    the step-1 corrector is negative in 46 cells); the library latches the
    error and returns it from
    the next synchronising call.  A stable deck latches nothing (every other
    test syncs)."""
    from paper_conf_cluster_regulymg15_b200 import CloverError
    deck = bm_deck(64)
    deck.update(max_timestep=10.0, initial_timestep=2.0, dtc_safe=14.0, dtu_safe=10.0,
                dtv_safe=10.0, dtdiv_safe=14.0)
    g = make_gpu(deck)
    g.step(1)
    with pytest.raises(CloverError) as ei:
        g.sync()
    assert ei.value.code == -6
    # a NaN in the state: the summary reports it, and the next step latches it
    g2 = make_gpu(bm_deck(64))
    rho = g2.read("density0")
    rho[20, 30] = np.nan
    g2.write("density0", rho)
    with pytest.raises(CloverError) as ei:
        g2.field_summary()
    assert ei.value.code == -8
    g2.step(1)
    with pytest.raises(CloverError) as ei:
        g2.sync()
    assert ei.value.code == -6


def test_y_wall_fold_guard(torch_cuda, monkeypatch):
    """the y-wall bands ride on a fixup launch only when all its
    blocks are co-resident.  Forcing the separate band launch gives the same
    bits (one launch more per step)."""
    deck = fuzz_deck(6, nx=96, ny=80)
    a = make_gpu(deck)
    monkeypatch.setenv("CLOVER_WALLS_FOLD_LIMIT", "0")
    b = make_gpu(deck)
    assert b.kernels_per_step() == a.kernels_per_step() + 1
    a.step(6)
    b.step(6)
    for f in STATE:
        assert np.array_equal(a.read(f), b.read(f)), f


def test_c2_960_87_steps(torch_cuda):
    """configs[1]: clover_bm_short shape, full run; also the QA constant."""
    deck = bm_deck(960, end_step=87)
    g, o = make_gpu(deck), Oracle(deck)
    g.step(87)
    dts = o.step(87)
    assert np.array_equal(g.dt_history(1, 87), dts)
    gs, os_ = g.field_summary(), o.field_summary()
    assert_summary_close(gs, os_)
    assert abs(100.0 * gs["ke"] / 1.19316898756307 - 100.0) < 0.001
    assert_fields_equal(g, o, ctx="C2")
    print("C2 IEEE fixup warp segments:", g.debug_fix_count())


@pytest.mark.parametrize("n,steps", [(3840, 20), (7680, 2)])
def test_full_size_first_steps(torch_cuda, n, steps):
    """configs[2] (bm 3840^2) over its first 20 steps and configs[3]'s 7680^2
    strong-scaling base over 2 steps, one chunk, graphs, in the bench's launch
    configuration: every state field and the dt history bitwise (the oracle
    needs ~1.8 s per step at 3840^2, ~8 s at 7680^2)."""
    deck = bm_deck(n, end_step=300)
    g, o = make_gpu(deck), Oracle(deck)
    g.step(steps)
    dts = o.step(steps)
    assert np.array_equal(g.dt_history(1, steps), dts)
    assert_fields_equal(g, o, ctx=f"{n}")
    # the sequential oracle sum carries up to n*eps (3e-9) of its own
    # rounding at this size; compare with its compensated twin
    assert_summary_close(g.field_summary(), o.field_summary(compensated=True))


def test_read_field_window_matches_full_read(torch_cuda):
    """clover_read_field_window == the same window of clover_read_field, on
    local chunks (the window spans chunk boundaries) for every field kind."""
    deck = fuzz_deck(5, nx=70, ny=52)
    g = make_gpu(deck, px=2, py=3)
    g.step(3)
    for f in ("density0", "pressure", "xvel0", "yvel0", "vol_flux_x", "vol_flux_y"):
        full = g.read(f)
        for j0, k0, w, h in ((1, 1, 5, 7), (30, 12, 20, 25), (1, 1, full.shape[1], full.shape[0])):
            a = g.read_window(f, j0, k0, w, h)
            assert np.array_equal(a, full[k0 - 1:k0 - 1 + h, j0 - 1:j0 - 1 + w]), (f, j0, k0)
    from paper_conf_cluster_regulymg15_b200 import CloverError
    with pytest.raises(CloverError):
        g.read_window("density0", 60, 1, 20, 5)  # past nx = 70


def test_maximum_size_corner_window_bitwise(torch_cuda):
    """Maximum sizes (one chunk of 20480^2 = 419 M cells, 61 GB of fields):
    a blast in the corner of a huge mesh evolves bit for bit like the same
    blast on a small mesh with the same cell size (dx = 10/20480 = 2^-11, so
    the 256-cell domain [0, 0.125]^2 has exactly the same geometry), for as
    long as nothing from the small mesh's far walls can have reached the
    window: one step's stencil reaches < 8 cells, so after 10 steps the
    cells below 128 are untouched by walls 256 cells away.  dt is set by the
    blast on both (the quiescent far field has a smaller sound speed), so the
    dt histories are bitwise equal too.  The oracle runs the small mesh."""
    from workloads import _state
    n_big, n_small, steps = 20480, 256, 10
    dx = 10.0 / n_big
    assert dx == 2.0 ** -11
    blast = _state(1.0, 2.5, geometry="rectangle", xmin=0.0, xmax=64 * dx, ymin=0.0, ymax=32 * dx)
    big = bm_deck(n_big)
    big["states"] = [_state(0.2, 1.0), blast]
    small = bm_deck(n_small, xmax=n_small * dx, ymax=n_small * dx)
    small["states"] = [_state(0.2, 1.0), dict(blast)]
    g = make_gpu(big)
    g.step(steps)
    o = Oracle(small)
    dts = o.step(steps)
    assert np.array_equal(g.dt_history(1, steps), dts)
    w = 128
    for f in STATE:
        a = g.read_window(f, 1, 1, w, w)
        b = o.read(f)[:w, :w]
        assert np.array_equal(a, b), (f, rel_cell(a, b))
    # and the far field is exactly the untouched background
    far = g.read_window("density0", n_big - 63, n_big - 63, 64, 64)
    assert np.all(far == 0.2)
    g.close()


@pytest.mark.parametrize("pxy,batch,expected", [((1, 1), True, 8), ((3, 1), False, 28),
                                                ((1, 3), False, 27), ((3, 1), True, 12),
                                                ((1, 3), True, 11)])
def test_kernels_per_step(torch_cuda, monkeypatch, pxy, batch, expected):
    """Launches per step (bench.py's gpu_launches): one chunk runs visc_dt,
    Lagrangian and both fused sweeps with a fixup each, the y-wall bands
    riding on the fixup before the y sweep (8); several chunks launch the
    bands separately (+1 per chunk with a y wall) and finalise dt in
    k_dt_finalize (+1); chunk boundaries keep both fused sweeps.  One launch
    per chunk (CLOVER_BATCH=0): 3x1 = 3 * (4 + 2 + 3) + 1, 1x3 = (4 + 2 + 3)
    + (4 + 2 + 2) + (4 + 2 + 3) + 1; batched: 3x1 = 8 + 3 bands + 1, 1x3 =
    8 + 2 bands + 1."""
    px, py = pxy
    if not batch:
        monkeypatch.setenv("CLOVER_BATCH", "0")
    g = make_gpu(fuzz_deck(11), px=px, py=py)
    assert g.kernels_per_step() == expected
    # the engine's own launch counter (clover_launch_count, the bench's
    # gpu_launches) agrees, through graph launches and direct launches
    n0 = g.launch_count()
    g.step(3)
    assert g.launch_count() - n0 == 3 * expected
    g.set_graphs(False)
    g.step(2)
    assert g.launch_count() - n0 == 5 * expected
