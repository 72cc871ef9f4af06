"""GPU parity: libperm's CUDA path vs the oracle, bit-exact (tolerance 0).

Inputs come from workloads/ (seeded); expected values from oracle.apply_ref
(b[P(i)] = a[i]), compared as raw 32-bit words.
"""
import numpy as np
import pytest

import workloads as W
from oracle import apply as OA

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icpp_kasagini13_b200 import build
    build.build()
    import paper_conf_icpp_kasagini13_b200 as pkg
    return pkg


def dev(x: np.ndarray):
    return torch.from_numpy(x.view(np.int32)).cuda()


def host_words(t) -> np.ndarray:
    return t.cpu().numpy().view(np.uint32)


def run(P, p, a, **kw):
    # the parity tests exercise the scheduled passes on every family: the
    # low-distribution shortcut (identity, shuffle) is tested on its own below
    kw.setdefault("direct", -1)
    with P.Plan(p, **kw) as plan:
        da = dev(a)
        db = torch.full_like(da, -1)
        plan.apply(da, db)
        torch.cuda.synchronize()
        return host_words(db), plan.info()


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k", [10, 12, 13, 14])
def test_fused_single_cta(P, fam, k):
    n = 1 << k
    p = W.make_perm(fam, n, seed=100 + k)
    a = W.make_data(n)
    b, info = run(P, p, a)
    assert info["passes"] == 1
    assert np.array_equal(b, OA.apply_ref(p, a))


def test_config0_bitrev_4096(P):
    # BASELINE configs[0]: n = 4096 (64 x 64) bit-reversal, bit-exact against the oracle
    n = 4096
    p = W.bitrev(n)
    a = W.make_data(n)
    for passes in (0, 3, 5):
        b, info = run(P, p, a, passes=passes)
        assert (info["rows"], info["cols"]) == (64, 64)
        assert np.array_equal(b, OA.apply_ref(p, a)), passes


@pytest.mark.parametrize("passes", [3, 5])
@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k", [12, 15, 16, 17, 19, 20])
def test_multi_pass(P, passes, fam, k):
    n = 1 << k
    p = W.make_perm(fam, n, seed=7 + k)
    a = W.make_data(n)
    b, info = run(P, p, a, passes=passes)
    assert info["passes"] == passes
    assert np.array_equal(b, OA.apply_ref(p, a))


@pytest.mark.parametrize("h", [(1, 4, 1), (4, 4, 4), (8, 8, 8), (2, 16, 2), (16, 32, 4), (4, 8, 16)])
def test_tile_shapes_tiled_layout(P, h):
    n = 1 << 18
    p = W.random(n, 3)
    a = W.make_data(n)
    b, info = run(P, p, a, passes=3, h=h, layout=1)
    assert info["h"] == list(h)
    assert np.array_equal(b, OA.apply_ref(p, a))


@pytest.mark.parametrize("fam", W.FAMILIES)
def test_config1_4M_all_families(P, fam):
    # BASELINE configs[1]: n = 2^22 float32, the five families of the paper (L373-L389)
    n = 1 << 22
    p = W.make_perm(fam, n)
    a = W.make_data(n)
    b, info = run(P, p, a)
    assert np.array_equal(b, OA.apply_ref(p, a))
    # the conventional kernels agree too
    da, dp = dev(a), torch.from_numpy(p).cuda()
    db = torch.empty_like(da)
    P.scatter_baseline(dp, da, db)
    torch.cuda.synchronize()
    assert np.array_equal(host_words(db), OA.apply_ref(p, a))
    dq = torch.from_numpy(OA.inverse(p)).cuda()
    db2 = torch.empty_like(da)
    P.gather_baseline(dq, da, db2)
    torch.cuda.synchronize()
    assert np.array_equal(host_words(db2), OA.apply_ref(p, a))


def test_config1_random_seeds_and_5pass(P):
    n = 1 << 22
    a = W.make_data(n)
    for seed in (42, 43, 44):
        p = W.random(n, seed)
        for passes, no_tma in ((3, 0), (5, 0), (5, 1)):
            b, _ = run(P, p, a, passes=passes, no_tma=no_tma)
            assert np.array_equal(b, OA.apply_ref(p, a)), (seed, passes)


@pytest.mark.parametrize("k", [21, 23, 24])
def test_odd_and_larger_views(P, k):
    n = 1 << k
    p = W.random(n, k)
    a = W.make_data(n)
    b, _ = run(P, p, a)
    assert np.array_equal(b, OA.apply_ref(p, a))


def test_config2_2pow26_random(P):
    # BASELINE configs[2]: n = 2^26 random, the launch configuration bench.py times
    n = 1 << 26
    p = W.random(n, 42)
    a = W.make_data(n)
    b, info = run(P, p, a)
    assert info["passes"] == 5
    assert np.array_equal(b, OA.apply_ref(p, a))
    b, info = run(P, p, a, passes=3)
    assert np.array_equal(b, OA.apply_ref(p, a))


def test_adversarial_payloads(P):
    n = 1 << 16
    a = np.array([0x7FC00001, 0xFFFFFFFF, 0x80000000, 0x00000001, 0x7F800000, 0xFF800000,
                  0x00000000, 0x7FBFFFFF] * (n // 8), dtype=np.uint32)
    a ^= np.arange(n, dtype=np.uint32) << np.uint32(20)
    for fam in W.FAMILIES:
        p = W.make_perm(fam, n)
        b, _ = run(P, p, a)
        assert np.array_equal(b, OA.apply_ref(p, a))


def test_repeated_apply_and_streams(P):
    n = 1 << 20
    p = W.random(n, 9)
    a = W.make_data(n)
    ref = OA.apply_ref(p, a)
    with P.Plan(p) as plan:
        da = dev(a)
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            outs = []
            for _ in range(3):
                db = torch.empty_like(da)
                plan.apply(da, db, stream=s)
                outs.append(db)
        s.synchronize()
        for db in outs:
            assert np.array_equal(host_words(db), ref)


def test_apply_host_e2e(P):
    n = 1 << 22
    p = W.random(n, 5)
    a = W.make_data(n)
    b = np.empty_like(a)
    with P.Plan(p) as plan:
        plan.apply_host(a, b)
    assert np.array_equal(b, OA.apply_ref(p, a))


def test_apply_host_async_two_streams(P):
    # perm_apply_host_async: several plans' host round trips enqueued on two streams
    # (copy engines of both directions overlap), results valid after the synchronisation
    ks = [(20, "random"), (21, "bitrev"), (22, "transpose"), (22, "random")]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    plans, bufs, refs = [], [], []
    for i, (k, fam) in enumerate(ks):
        n = 1 << k
        p = W.make_perm(fam, n, seed=30 + i)
        a = W.make_data(n, seed=60 + i)
        ha = torch.from_numpy(a.view(np.int32)).pin_memory()
        hb = torch.empty(n, dtype=torch.int32).pin_memory()
        plans.append(P.Plan(p))
        bufs.append((ha, hb))
        refs.append(OA.apply_ref(p, a))
    for i, pl in enumerate(plans):
        pl.apply_host_async(bufs[i][0], bufs[i][1], streams[i % 2])
    torch.cuda.synchronize()
    for i, pl in enumerate(plans):
        assert np.array_equal(bufs[i][1].numpy().view(np.uint32), refs[i]), ks[i]
        pl.close()
    with pytest.raises(P.PermError):          # pageable memory is refused by the binding
        with P.Plan(W.random(1 << 12, 1)) as pl:
            x = torch.zeros(1 << 12, dtype=torch.int32)
            pl.apply_host_async(x, x.clone())


def test_profiling_pass_times(P):
    n = 1 << 22
    with P.Plan(W.random(n, 1)) as plan:
        da = torch.zeros(n, dtype=torch.int32, device="cuda")
        db = torch.empty_like(da)
        plan.set_profiling(True)
        plan.apply(da, db)
        t = plan.pass_times()
        assert len(t) == plan.info()["kernels_per_apply"] and all(x > 0 for x in t)


def test_apply_errors(P):
    n = 1 << 16
    with P.Plan(W.random(n, 1)) as plan:
        da = torch.zeros(n + 16, dtype=torch.int32, device="cuda")
        with pytest.raises(P.PermError) as e:
            plan.apply(da, da)                      # aliasing
        assert e.value.status == -1
        with pytest.raises(P.PermError) as e:
            plan.apply(da[4:], da[4 + n // 2:])     # overlapping
        assert e.value.status == -1
        with pytest.raises(P.PermError) as e:
            plan.apply(da[1:], torch.empty_like(da))  # misaligned
        assert e.value.status == -1


def test_copy_kernel(P):
    a = dev(W.make_data(1 << 20))
    b = torch.empty_like(a)
    P.copy_kernel(a, b)
    torch.cuda.synchronize()
    assert torch.equal(a, b)


@pytest.mark.parametrize("layout", [3])
@pytest.mark.parametrize("k", [16, 18, 20, 22])
def test_fused3_first_apply_and_graph_replay(P, k, layout):
    # the single-launch 3-pass kernel: grid barriers must hold on the FIRST apply of a
    # fresh plan (intermediates not yet valid), for grids with idle CTAs (few tiles),
    # and across CUDA-graph replays (self-resetting counters)
    n = 1 << k
    p = W.random(n, 100 + k)
    a = W.make_data(n)
    ref = OA.apply_ref(p, a)
    with P.Plan(p, layout=layout, fuse=1) as plan:
        info = plan.describe()
        da = dev(a)
        db = torch.full_like(da, -1)
        plan.apply(da, db)
        torch.cuda.synchronize()
        assert info.get("fused3") == 1
        assert np.array_equal(host_words(db), ref)
        s = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            plan.apply(da, db, stream=s)
        for _ in range(3):
            db.fill_(-1)
            g.replay()
            torch.cuda.synchronize()
            assert np.array_equal(host_words(db), ref)


@pytest.mark.parametrize("layout", [1, 3])
@pytest.mark.parametrize("k", [16, 19, 20, 22])
def test_every_layout(P, layout, k):
    n = 1 << k
    p = W.random(n, 300 + k)
    a = W.make_data(n)
    ref = OA.apply_ref(p, a)
    for fam_p in (p, W.bitrev(n)):
        b, info = run(P, fam_p, a, passes=3, layout=layout)
        assert np.array_equal(b, OA.apply_ref(fam_p, a)), (layout, k)


@pytest.mark.parametrize("k", [10, 13, 16, 19, 21, 23])
def test_fp64_elements(P, k):
    # Table II(b): float64 payloads (raw 64-bit words), every family
    n = 1 << k
    a = W.make_data(n, 8)
    for fam in W.FAMILIES:
        p = W.make_perm(fam, n, seed=k)
        with P.Plan(p, elem_bytes=8, direct=-1) as plan:
            da = torch.from_numpy(a.view(np.int64)).cuda()
            db = torch.full_like(da, -1)
            plan.apply(da, db)
            torch.cuda.synchronize()
            got = db.cpu().numpy().view(np.uint64)
        assert np.array_equal(got, OA.apply_ref(p, a)), (fam, k)
    # conventional kernels on 8-byte elements
    p = W.random(n, 1)
    da = torch.from_numpy(a.view(np.int64)).cuda()
    db = torch.empty_like(da)
    P.scatter_baseline(torch.from_numpy(p).cuda(), da, db, elem_bytes=8)
    torch.cuda.synchronize()
    assert np.array_equal(db.cpu().numpy().view(np.uint64), OA.apply_ref(p, a))
    P.gather_baseline(torch.from_numpy(OA.inverse(p)).cuda(), da, db, elem_bytes=8)
    torch.cuda.synchronize()
    assert np.array_equal(db.cpu().numpy().view(np.uint64), OA.apply_ref(p, a))


@pytest.mark.parametrize("k", [10, 14, 16, 22])
@pytest.mark.parametrize("eb", [4, 8])
def test_direct_shortcut(P, k, eb):
    # for D_w(P) <= 2n/w (identical, shuffle) one coalesced kernel
    # is the faster choice; the plan takes it by default (S-designated on q = P^-1,
    # direct 1; D-designated on p with direct 2) and stays bit-exact
    n = 1 << k
    a = W.make_data(n, eb)
    view = np.int32 if eb == 4 else np.int64
    for fam, direct, want in (("identity", 0, 3), ("shuffle", 0, 1), ("random", 0, 0),
                              ("random", 1, 1), ("bitrev", 1, 1), ("identity", -1, 0),
                              ("shuffle", 2, 2), ("random", 2, 2), ("identity", 1, 1),
                              ("blocks", 0, 3)):
        if fam == "blocks":   # whole aligned 32-word blocks moved in order (direct 3)
            blocks = np.random.default_rng(k).permutation(n // 32).astype(np.int32)
            p = (blocks[:, None] * 32 + np.arange(32, dtype=np.int32)).reshape(-1)
        else:
            p = W.make_perm(fam, n, seed=k)
        with P.Plan(p, elem_bytes=eb, direct=direct) as plan:
            info = plan.info()
            assert info["direct"] == want, (fam, direct)
            if want:
                assert info["kernels_per_apply"] == 1
            da = torch.from_numpy(a.view(view)).cuda()
            db = torch.full_like(da, -1)
            plan.apply(da, db)
            torch.cuda.synchronize()
            got = db.cpu().numpy().view(a.dtype)
        assert np.array_equal(got, OA.apply_ref(p, a)), (fam, direct, k, eb)


# TLC ring configurations: tiles per CTA > A slots and > B slots, so both rings wrap
# (a missing async-proxy fence before a slot's TMA refill only shows up then)
@pytest.mark.parametrize("k,h,stages,fuse,log2c", [
    (20, (16, 16, 16), 1, 0, 0),      # EPT 32, NA 1, NB 1
    (20, (8, 8, 8), 1, 0, 0),         # EPT 16, NA 1, NB 2
    (22, (8, 8, 8), 0, 0, 0),         # EPT 32, NA 2, NB 1, ~2 tiles per CTA
    (22, (2, 4, 2), 0, 0, 0),         # EPT 8 / 16 / 8, NA 6, ~7 tiles per CTA, 32-byte chunks
    (22, (2, 2, 2), 0, 0, 0),         # rejected: h2 < 4
    (22, (4, 4, 4), 2, 1, 0),         # fused single launch, NA 2
    (24, (4, 4, 4), 0, 0, 0),         # EPT 32, ~7 tiles per CTA
    (24, (4, 4, 4), 0, 1, 0),
    (24, (1, 4, 1), 0, 0, 13),        # non-square view 2048 x 8192, 16-byte chunks
])
def test_tlc_rings_wrap(P, k, h, stages, fuse, log2c):
    n = 1 << k
    p = W.random(n, 77 + k)
    a = W.make_data(n)
    try:
        b, info = run(P, p, a, passes=3, layout=3, h=h, stages=stages, fuse=fuse, log2c=log2c)
    except P.PermError as e:
        assert h[1] < 4 and "h" in str(e)      # h2 >= 4 (16-byte tensor-store rows)
        return
    assert np.array_equal(b, OA.apply_ref(p, a)), (k, h, stages, fuse, log2c)


@pytest.mark.parametrize("fmt", [-1, 0, 1])
@pytest.mark.parametrize("k", [15, 17, 20, 21, 22, 23, 25])
def test_tlc_entry_formats(P, k, fmt):
    # full (source row << log2 tile | destination) vs compact (line index implied) entries
    n = 1 << k
    p = W.random(n, 500 + k)
    a = W.make_data(n)
    b, info = run(P, p, a, passes=3, layout=3, sched_format=fmt)
    assert np.array_equal(b, OA.apply_ref(p, a)), (k, fmt, info["entry_bits"])


@pytest.mark.parametrize("k", [16, 22])
def test_run_pass_chain_is_apply(P, k):
    # perm_plan_run_pass (diagnostics / roofline timing): the three passes launched one by
    # one through the plan's own intermediates give exactly b[P(i)] = a[i]
    n = 1 << k
    p = W.random(n, 900 + k)
    a = W.make_data(n)
    with P.Plan(p, passes=3) as plan:
        da = dev(a)
        db = torch.full_like(da, -1)
        plan.run_pass(0, da)
        plan.run_pass(1, None)
        plan.run_pass(2, None, db)
        torch.cuda.synchronize()
        assert np.array_equal(host_words(db), OA.apply_ref(p, a))
        with pytest.raises(P.PermError):
            plan.run_pass(3, da)


@pytest.mark.parametrize("fam", ["random", "bitrev", "transpose"])
@pytest.mark.parametrize("k", [12, 16, 19, 22])
def test_schedule_from_global(P, fam, k):
    # 5-pass TMA row passes whose slots hold the data only; the permuters read the
    # schedule from global memory (the default for lines of >= 16384 words, n >= 2^27)
    n = 1 << k
    p = W.make_perm(fam, n, seed=11 + k)
    a = W.make_data(n)
    ref = OA.apply_ref(p, a)
    for stages in (0, 1, 3):
        b, info = run(P, p, a, passes=5, no_tma=-1, stages=stages)
        assert info["passes"] == 5
        assert np.array_equal(b, ref), stages
    # dense schedule bitstreams (default for L >= 16384) in the SG, slot and plain kernels
    for no_tma in (-1, 0, 1):
        b, _ = run(P, p, a, passes=5, no_tma=no_tma, sched_format=2)
        assert np.array_equal(b, ref), ("dense", no_tma)


@pytest.mark.parametrize("fam,k", [(f, k) for f in ("random", "bitrev", "identity") for k in (16, 20, 22, 24)]
                         + [("random", 26)])
def test_half_line_ring(P, fam, k):
    # 5-pass row passes on the ring of three half-line slots (the default for lines of
    # 32768 words, n = 2^29..2^30), forced here at small n: one line per CTA, the two
    # halves of a line in any two slots, loads overlapping the permute and the stores
    n = 1 << k
    p = W.make_perm(fam, n, seed=31 + k)
    a = W.make_data(n)
    for fmt in (-1, 2):          # W64 and dense schedule formats
        with P.Plan(p, passes=5, no_tma=-2, direct=-1, sched_format=fmt) as plan:
            d = plan.describe()
            assert all(rp["split"] == 1 and rp["h"] == 1 for rp in d["row_passes"])
            assert all(rp["dense"] == (fmt == 2) for rp in d["row_passes"])
            da = dev(a)
            db = torch.full_like(da, -1)
            plan.apply(da, db)
            torch.cuda.synchronize()
            assert np.array_equal(host_words(db), OA.apply_ref(p, a)), fmt


@pytest.mark.parametrize("k", [19, 21])
@pytest.mark.parametrize("fam", ["random", "transpose", "bitrev"])
def test_tall_views_5pass(P, k, fam):
    # r > c views (the n = 2^29 default shape, L603: the view need not be square)
    n = 1 << k
    p = W.make_perm(fam, n, seed=k)
    a = W.make_data(n)
    b, info = run(P, p, a, passes=5, log2c=k // 2)
    assert (info["rows"], info["cols"]) == (1 << (k - k // 2), 1 << (k // 2))
    assert np.array_equal(b, OA.apply_ref(p, a))


@pytest.mark.parametrize("k,log2c", [(19, 14), (20, 15), (21, 15)])
@pytest.mark.parametrize("fam", ["random", "bitrev"])
def test_half_line_ring_staged_schedule(P, k, log2c, fam):
    # the half-line ring with the schedule streamed through shared memory in TMA chunks
    # (lines of 16384 / 32768 words via wide views, L603)
    n = 1 << k
    p = W.make_perm(fam, n, seed=k + log2c)
    a = W.make_data(n)
    ref = OA.apply_ref(p, a)
    for fmt in (-1, 0):           # W64 chunks (4 x 8 KiB) and dense chunks (5 x 64*E words)
        with P.Plan(p, passes=5, no_tma=-2, direct=-1, log2c=log2c, sched_format=fmt) as plan:
            d = plan.describe()
            long_lines = [rp for rp in d["row_passes"] if rp["L"] >= 16384]
            assert long_lines and all(rp["threads"] == 512 for rp in long_lines)
            assert all(rp["dense"] == (fmt == 0) for rp in long_lines)
            da = dev(a)
            db = torch.full_like(da, -1)
            plan.apply(da, db)
            torch.cuda.synchronize()
            assert np.array_equal(host_words(db), ref), fmt


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k,C", [(15, 8), (15, 16), (16, 8), (16, 16), (17, 16), (18, 16), (16, 2), (17, 4)])
def test_cluster_path(P, fam, k, C):
    # NEXT-4: one launch of one thread-block cluster; the column phase's
    # transposes are DSMEM block exchanges; bit-exact against the definition
    n = 1 << k
    p = W.make_perm(fam, n, seed=k * C)
    a = W.make_data(n)
    try:
        b, info = run(P, p, a, passes=2, cluster=C)
    except P.PermError as e:
        # a cluster of C blocks with 3 * n/C words each must fit the GPU (C = 2: 2^16 only)
        assert e.status in (-1, -3), e
        return
    assert info["passes"] == 2 and info["kernels_per_apply"] == 1
    assert np.array_equal(b, OA.apply_ref(p, a)), (fam, k, C)


def test_cluster_path_fp64_and_replay(P):
    n = 1 << 16
    p = W.random(n, 77)
    a = W.make_data(n, elem_bytes=8)
    with P.Plan(p, elem_bytes=8, passes=2, direct=-1) as plan:
        da = torch.from_numpy(a.view(np.int32)).cuda()
        db = torch.full_like(da, -1)
        for _ in range(3):                       # repeated launches (fresh shared memory each)
            plan.apply(da, db)
        torch.cuda.synchronize()
        assert np.array_equal(db.cpu().numpy().view(np.uint64), OA.apply_ref(p, a))


@pytest.mark.parametrize("fam", ["random", "bitrev", "transpose", "shuffle"])
@pytest.mark.parametrize("k", [20, 21, 22, 26])
def test_tlc_ring(P, fam, k):
    # layout 5: the TLC passes (transposes absorbed into X1 / X2 chunks) with 32768-word
    # tiles permuted in place through the half-tile ring, chunked tensor stores per half
    n = 1 << k
    p = W.make_perm(fam, n, seed=k + 5)
    a = W.make_data(n)
    b, info = run(P, p, a, layout=5)
    assert info["passes"] == 3 and info["entry_bits"] == [25, 25, 25]
    assert np.array_equal(b, OA.apply_ref(p, a)), (fam, k)
