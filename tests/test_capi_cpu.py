"""CPU-side tests of libperm: the library loads, exports every symbol the header
declares, validates its inputs, and its C++ planner's exported plans satisfy
the oracle's invariants (i)-(vii) — checked by oracle/check.py, which shares
no code with the planner — and drive the paper-faithful emulator to b[P(i)] = a[i].
No compute call touches a GPU here (perm_plan_create_host)."""
import ctypes
import os
import re

import numpy as np
import pytest

import workloads as W
from oracle import apply as OA
from oracle import check as OC
from oracle import emulate as OE

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_icpp_kasagini13_b200 import build
    build.build()
    import paper_conf_icpp_kasagini13_b200 as P
    return P


def header_functions():
    txt = open(os.path.join(ROOT, "include", "perm.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(perm_[a-z_0-9]+)\s*\(", txt)))


def test_exports_every_declared_symbol(lib):
    names = header_functions()
    assert "perm_plan_create" in names and "perm_apply" in names and "perm_plan_destroy" in names
    so = ctypes.CDLL(lib.LIB_PATH)
    missing = [n for n in names if not hasattr(so, n)]
    assert not missing, missing


def test_library_is_sm100a(lib):
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", lib.LIB_PATH], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def decode(sched):
    s = np.asarray(sched, dtype=np.uint32)
    return (s >> 16).astype(np.int64), (s & 0xFFFF).astype(np.int64)


def export_plan(lib, p, **kw):
    kw.setdefault("direct", -1)     # shortcut plans (identity, shuffle) have no schedule
    with lib.Plan(p, device=False, **kw) as pl:
        info = pl.info()
        kappa, scheds = pl.export()
    return info, kappa.astype(np.int64), [decode(s) for s in scheds]


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k", [10, 11, 12, 13, 14, 15, 16])
def test_cpp_plan_passes_oracle_checker(lib, fam, k):
    n = 1 << k
    p = W.make_perm(fam, n, seed=42 + k)
    info, kappa, sched = export_plan(lib, p, passes=5 if k >= 15 else 0)   # per-line schedules
    r, c = W.view_shape(n)
    assert (info["rows"], info["cols"]) == (r, c)
    OC.assert_plan(p, kappa, sched, r, c, 32)
    for f, L in enumerate((c, r, c)):
        assert info["entry_bits"][f] == 2 * (L.bit_length() - 1) - 5


@pytest.mark.parametrize("k", [12, 13])
def test_cpp_plan_drives_emulator(lib, k):
    n = 1 << k
    r, c = W.view_shape(n)
    a = W.make_data(n)
    for fam in W.FAMILIES:
        p = W.make_perm(fam, n)
        _, kappa, sched = export_plan(lib, p)
        b, rc = OE.scheduled(a, sched, r, c, 32)
        assert np.array_equal(b, OA.apply_ref(p, a))
        t = rc.table()
        assert t[("global", "read", "coalesced")] == 11 and t[("global", "write", "coalesced")] == 5
        assert t[("shared", "read", "conflict-free")] == 8
        assert t[("shared", "write", "conflict-free")] == 8


@pytest.mark.parametrize("k", [18, 20])
def test_cpp_plan_larger(lib, k):
    n = 1 << k
    r, c = W.view_shape(n)
    for fam in ("random", "bitrev"):
        p = W.make_perm(fam, n)
        _, kappa, sched = export_plan(lib, p, passes=5)
        OC.assert_plan(p, kappa, sched, r, c, 32)


def test_cpp_plan_22_random(lib):
    n = 1 << 22
    r, c = W.view_shape(n)
    p = W.random(n, 42)
    info, kappa, sched = export_plan(lib, p, passes=5)
    OC.assert_plan(p, kappa, sched, r, c, 32)
    assert info["passes"] == 5
    # W64 schedule: 17-bit entries, 3 per 64-bit word, 11 words per warp-round of 32
    assert info["entry_bits"] == [17, 17, 17]
    assert info["sched_bytes"] == 3 * ((n // 32) * 11 * 8 + 16)    # + 4 pad words per phase


def test_pass_options_and_info(lib):
    n = 1 << 16
    p = W.random(n, 1)
    for passes in (3, 5):
        with lib.Plan(p, device=False, passes=passes) as pl:
            info = pl.info()
            assert info["passes"] == passes
            assert info["kernels_per_apply"] in (1, passes)   # 1 = single persistent launch
    with lib.Plan(W.random(1 << 12, 1), device=False) as pl:
        assert pl.info()["passes"] == 1
    with lib.Plan(p, device=False, passes=3, layout=1, h=(4, 8, 4)) as pl:
        assert pl.info()["h"] == [4, 8, 4]


def test_errors(lib):
    with pytest.raises(lib.PermError) as e:
        lib.Plan(np.array([0, 0] + list(range(2, 1024)), dtype=np.int32), device=False)
    assert e.value.status == -2
    with pytest.raises(lib.PermError) as e:
        lib.Plan(np.arange(1000, dtype=np.int32), device=False)
    assert e.value.status == -3
    with pytest.raises(lib.PermError) as e:
        lib.Plan(np.arange(1024, dtype=np.int32), elem_bytes=2, device=False)
    assert e.value.status == -3
    bad = np.arange(1024, dtype=np.int32)
    bad[5] = 1024
    with pytest.raises(lib.PermError) as e:
        lib.Plan(bad, device=False)
    assert e.value.status == -2
    with pytest.raises(lib.PermError) as e:
        lib.Plan(W.random(1 << 16, 1), device=False, passes=3, h=(4, 3, 4))
    assert e.value.status == -1
    # a host-only plan cannot apply
    with lib.Plan(W.random(1 << 12, 1), device=False) as pl:
        with pytest.raises(lib.PermError) as e:
            pl.apply(1 << 20, 2 << 20, stream=0)
        assert e.value.status == -7


def test_bruteforce_tiny_via_cpp_euler_split(lib):
    # the smallest view the library supports is 32 x 32; exhaustively permute
    # one 8-element block of rows inside an otherwise random permutation
    import itertools
    n = 1 << 10
    base = W.random(n, 5)
    r, c = W.view_shape(n)
    for perm in itertools.islice(itertools.permutations(range(8)), 0, 40320, 97):
        p = base.copy()
        p[:8] = base[list(perm)]
        _, kappa, sched = export_plan(lib, p)
        OC.assert_plan(p, kappa, sched, r, c, 32)


# ---------------------------------------------------------------- TLC plans (layout 3)

def export_tlc(lib, p, **kw):
    kw.setdefault("direct", -1)
    with lib.Plan(p, device=False, passes=3, layout=3, **kw) as pl:
        info = pl.info()
        d = pl.describe()
        kappa, scheds = pl.export()
    return info, d, kappa.astype(np.int64), [s.reshape(-1) for s in scheds]


@pytest.mark.parametrize("fam", W.FAMILIES)
@pytest.mark.parametrize("k", [16, 17, 18, 20])
def test_tlc_plan_passes_oracle_checker(lib, fam, k):
    n = 1 << k
    r, c = W.view_shape(n)
    p = W.make_perm(fam, n, seed=k)
    info, d, kappa, sched = export_tlc(lib, p)
    h = tuple(info["h"])
    res = OC.check_tlc(p, kappa, sched, r, c, h)
    assert all(res.values()), res
    assert len(res) == 8


def test_tlc_plan_22(lib):
    n = 1 << 22
    r, c = W.view_shape(n)
    p = W.random(n, 42)
    info, d, kappa, sched = export_tlc(lib, p)
    assert info["h"] == [4, 4, 4] and info["entry_bits"] == [21, 21, 21]
    # compact entries: sigma (8 bits) + destination position in the line (11 bits)
    info_c, _, kappa_c, sched_c = export_tlc(lib, p, sched_format=1)
    assert info_c["entry_bits"] == [19, 19, 19]
    res = OC.check_tlc(p, kappa_c, sched_c, r, c, (4, 4, 4))
    assert all(res.values()), res
    res = OC.check_tlc(p, kappa, sched, r, c, (4, 4, 4))
    assert all(res.values()), res


@pytest.mark.parametrize("k", [20, 21, 22])
def test_tlc_full_and_compact_formats_agree(lib, k):
    # the two device entry formats must export the same logical (src, dst) schedule
    # (compact kernels are compiled for 8192- and 16384-word tiles, i.e. n >= 2^20)
    n = 1 << k
    r, c = W.view_shape(n)
    p = W.make_perm("random", n, seed=k)
    # 8192-word tiles (the default at 2^21 is 4096-word tiles, which have no compact kernel)
    h = (4, 8, 4) if k == 21 else (0, 0, 0)
    i_full, _, kappa_f, s_full = export_tlc(lib, p, sched_format=-1, h=h)
    i_cmp, _, kappa_c, s_cmp = export_tlc(lib, p, sched_format=1, h=h)
    assert np.array_equal(kappa_f, kappa_c)
    for a, b in zip(s_full, s_cmp):
        assert np.array_equal(a, b)
    assert all(ec <= ef for ec, ef in zip(i_cmp["entry_bits"], i_full["entry_bits"]))
    assert i_cmp["entry_bits"][0] < i_full["entry_bits"][0]
    assert i_cmp["sched_bytes"] < i_full["sched_bytes"]
    res = OC.check_tlc(p, kappa_c, s_cmp, r, c, tuple(i_cmp["h"]))
    assert all(res.values()), res


@pytest.mark.parametrize("k,log2c,h", [(16, 10, (0, 0, 0)), (16, 6, (0, 0, 0)), (18, 12, (1, 64, 1)),
                                         (19, 12, (2, 64, 2))])
def test_tlc_non_square_view(lib, k, log2c, h):
    # the r x c view "is not restricted to a square matrix"
    n = 1 << k
    r, c = n >> log2c, 1 << log2c
    p = W.make_perm("random", n, seed=k)
    info, d, kappa, sched = export_tlc(lib, p, log2c=log2c, h=h)
    assert (info["rows"], info["cols"]) == (r, c)
    res = OC.check_tlc(p, kappa, sched, r, c, tuple(info["h"]))
    assert all(res.values()), res


def test_tlc_checker_rejects_corruption(lib):
    n = 1 << 16
    r, c = W.view_shape(n)
    p = W.random(n, 7)
    info, d, kappa, sched = export_tlc(lib, p)
    h = tuple(info["h"])
    assert all(OC.check_tlc(p, kappa, sched, r, c, h).values())
    bad = [s.copy() for s in sched]
    # swap the destinations of two slots of one round: still a bijection, wrong mapping
    bad[1][0], bad[1][1] = (bad[1][0] & 0xFFFF0000) | (bad[1][1] & 0xFFFF), (bad[1][1] & 0xFFFF0000) | (bad[1][0] & 0xFFFF)
    res = OC.check_tlc(p, kappa, bad, r, c, h)
    assert not res["v_tiles_implement_phi"]
    # move a slot's source into another lane's bank
    bad = [s.copy() for s in sched]
    bad[2][0] = ((((bad[2][0] >> 16) ^ 1)) << 16) | (bad[2][0] & 0xFFFF)
    res = OC.check_tlc(p, kappa, bad, r, c, h)
    assert not (res["viii_lane_is_source_bank"] and res["vii_sources_and_dests_cover_tile"])


@pytest.mark.parametrize("k", [10, 13, 16, 19])
def test_fp64_plan_is_the_word_pair_permutation(lib, k):
    # Table II(b) (L731-L755): 8-byte elements; element i = words (2i, 2i+1) -> 2P(i)+h
    n = 1 << k
    p = W.random(n, k)
    with lib.Plan(p, elem_bytes=8, device=False, passes=5 if k >= 14 else 0) as pl:
        info = pl.info()
        kappa, sched = pl.export()
    assert info["elem_bytes"] == 8 and info["n"] == n
    p2 = np.empty(2 * n, dtype=np.int64)
    p2[0::2] = 2 * p.astype(np.int64)
    p2[1::2] = 2 * p.astype(np.int64) + 1
    r, c = W.view_shape(2 * n)
    OC.assert_plan(p2, kappa.astype(np.int64), [decode(s) for s in sched], r, c, 32)


def test_fp64_errors(lib):
    with pytest.raises(lib.PermError) as e:
        lib.Plan(np.array([0, 0] + list(range(2, 1024)), dtype=np.int32), elem_bytes=8, device=False)
    assert e.value.status == -2


def test_planner_is_deterministic_across_thread_counts(lib):
    # sharded ranks colour P independently and must agree exactly (the parallel Euler
    # split canonicalises every cycle's polarity and does not chunk by thread count)
    import subprocess, sys, json
    n = 1 << 21
    code = (
        "import sys, hashlib; sys.path.insert(0, %r)\n"
        "import workloads as W, paper_conf_icpp_kasagini13_b200 as P\n"
        "pl = P.Plan(W.random(%d, 3), device=False, passes=5)\n"
        "k, s = pl.export()\n"
        "print(hashlib.sha256(k.tobytes() + b''.join(x.tobytes() for x in s)).hexdigest())\n"
    ) % (ROOT, n)
    digests = set()
    for threads in ("1", "3", "8"):
        env = dict(os.environ, OMP_NUM_THREADS=threads)
        out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env)
        assert out.returncode == 0, out.stderr
        digests.add(out.stdout.strip())
    assert len(digests) == 1


@pytest.mark.parametrize("k", [10, 14, 16])
def test_distribution_and_direct_shortcut(lib, k):
    # D_w(P) reported by the planner equals the oracle's (L389-L401); the shortcut
    # (L699-L701) is taken exactly when D_w(P) <= 2n/w unless forced either way
    from oracle import distribution as OD
    n = 1 << k
    for fam in W.FAMILIES:
        p = W.make_perm(fam, n, seed=k)
        dw = OD.distribution(p, 32)
        for eb in (4, 8):
            pp = p if eb == 4 else np.stack([2 * p, 2 * p + 1], axis=1).reshape(-1).astype(np.int32)
            want_dw = OD.distribution(pp, 32) if eb == 8 else dw
            with lib.Plan(p, elem_bytes=eb, device=False) as pl:
                inf = pl.info()
                assert inf["distribution"] == want_dw, (fam, eb)
                m = pp.size // 32
                blk = pp.reshape(m, 32)
                in_order = bool(np.all(blk == blk[:, :1] + np.arange(32)) and np.all(blk[:, 0] % 32 == 0))
                low = want_dw <= 2 * pp.size // 32
                assert inf["direct"] == (3 if low and in_order else int(low)), (fam, eb)
                assert pl.describe()["direct"] == inf["direct"]
        with lib.Plan(p, device=False, direct=-1) as pl:
            assert pl.info()["direct"] == 0
        with lib.Plan(p, device=False, direct=1) as pl:
            assert pl.info()["direct"] == 1
        with lib.Plan(p, device=False, direct=2) as pl:
            assert pl.info()["direct"] == 2
        # the S-designated shortcut on q = P^-1 relies on D_w(P^-1) = D_w(P): both
        # count the distinct (source warp block, destination group) pairs
        q = np.empty_like(p)
        q[p] = np.arange(n, dtype=p.dtype)
        assert OD.distribution(q, 32) == dw, fam
    # identity and shuffle are the paper's low-distribution cases
    assert lib.Plan(W.identity(n), device=False).info()["direct"] == 3
    blocks = np.random.default_rng(k).permutation(n // 32).astype(np.int32)
    pb = (blocks[:, None] * 32 + np.arange(32, dtype=np.int32)).reshape(-1)
    assert lib.Plan(pb, device=False).info()["direct"] == 3
    assert lib.Plan(W.identity(n), device=False, direct=1).info()["direct"] == 1
    assert lib.Plan(W.make_perm("shuffle", n), device=False).info()["direct"] == 1
    assert lib.Plan(W.make_perm("bitrev", n), device=False).info()["direct"] == 0
    if k >= 16:   # sharded plans never take the single-device shortcut
        assert lib.Plan(W.identity(n), device=False, world=2, rank=0).info()["direct"] == 0


@pytest.mark.parametrize("k", [12, 14, 16, 17])
@pytest.mark.parametrize("fam", ["random", "bitrev", "shuffle"])
def test_dense_schedule_format_passes_oracle_checker(lib, fam, k):
    # 5-pass per-line schedules as dense bitstreams (E bits per entry, the default for
    # lines of >= 16384 words; forced here with sched_format = 2) decode to a valid plan
    n = 1 << k
    r, c = W.view_shape(n)
    p = W.make_perm(fam, n, seed=5 + k)
    info, kappa, sched = export_plan(lib, p, passes=5, sched_format=2)
    OC.assert_plan(p, kappa, sched, r, c, 32)
    with lib.Plan(p, device=False, passes=5, sched_format=2, direct=-1) as pl:
        d = pl.describe()
    for rp in d["row_passes"]:
        assert rp["dense"] == 1 and rp["sched_words_per_line"] == rp["L"] // 32 * rp["E"]
    # W64 (sched_format = -1) and dense give the same logical schedule
    _, kappa2, sched2 = export_plan(lib, p, passes=5, sched_format=-1)
    assert np.array_equal(kappa, kappa2)
    for (s1, t1), (s2, t2) in zip(sched, sched2):
        assert np.array_equal(s1, s2) and np.array_equal(t1, t2)
