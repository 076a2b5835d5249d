"""Pins of the CPU oracle against what the paper and the mathematics fix.

Every expected value below is either a closed form derived by hand from the
construction of the input (cited to the paper passage the construction
follows), a textbook/library routine on a tiny input, or an O(n^2) brute
force -- never a re-run of the oracle's own formula.  SURVEY.md 8(c) "What
pins each part" maps each oracle definition (C1-C12) to these tests.
"""
import numpy as np
import pytest

from oracle import oracle as O
from gen import vegen as G
from tests.helpers import BF, F, S, U, f32, f64, le_bytes, meta, obj, records, zeros

CFG1_BASE = 0x7F0000000000


def _cfg1():
    objs = [dict(o, pre=G.snapshot_host(1, 0, 1, 0, 0), post=G.snapshot_host(1, 0, 1, 0, 1))
            for o in G.objects(1)]
    recs = G.records_host(1, 0, 1, 0, 1 << 20)
    cfg = O.make_config(16)
    return cfg, objs, recs


@pytest.fixture(scope="module")
def cfg1():
    cfg, objs, recs = _cfg1()
    keys, glob, objstat = O.analyze(cfg, objs, recs)
    return cfg, objs, recs, keys, glob, objstat


# --------------------------------------------------------------------------
# cfg1 closed forms (BASELINE.json configs[0]; SURVEY 8(d) "cfg1 PC roles")
# --------------------------------------------------------------------------

def test_cfg1_counts_and_globals(cfg1):
    cfg, objs, recs, keys, glob, objstat = cfg1
    assert glob["n_records"] == 1 << 20 and glob["n_invalid"] == 0 and glob["n_unmapped"] == 0
    for p in range(16):
        k = keys[p]
        if p < 8:
            assert (k["n_ld"], k["n_st"], k["n_ld_eq_pre"]) == (65536, 0, 65536)   # loads read pre
        else:
            assert (k["n_ld"], k["n_st"]) == (0, 65536)
        assert k["single_type"] == 1
    o = keys[16]
    assert o["n_ld"] == 8 * 65536 and o["n_st"] == 8 * 65536
    assert o["single_type"] == 0 and o["heavy"] == 255 and o["structured"] == 0 and o["approx"] == 0   # Q15
    assert objstat[0]["n_ld_reload"] == 0                                      # every element loaded once


def test_cfg1_pc_roles(cfg1):
    cfg, objs, recs, keys, glob, objstat = cfg1
    k = keys
    assert k[0]["single_zero"] and k[0]["n_zero"] == 65536                       # PC0 zero
    assert k[1]["single_value"] and k[1]["heavy"] == 0 and k[1]["dict8"]         # PC1 0x2A -> u8
    # PC2: 3e-7 over slice 2 -> exact line with the slice's end points
    assert k[2]["structured"] and k[2]["line_state"] == O.LINE_LINE
    assert k[2]["p_x"] == CFG1_BASE + 4 * 131072 and O.y_of(k[2]["p_ylo"], k[2]["p_yhi"]) == 3 * 131072 - 7
    assert k[2]["q_x"] == CFG1_BASE + 4 * 196607 and O.y_of(k[2]["q_ylo"], k[2]["q_yhi"]) == 3 * 196607 - 7
    assert k[3]["heavy"] == 4 and k[3]["n_distinct"] == 102                      # [-1,100] -> i8 (P5)
    assert k[4]["top_bits"][0] == 0x3F800000 and k[4]["top_count"][0] == 58982 and k[4]["frequent"]
    assert k[5]["approx"] and not k[5]["single_value"] and k[5]["n_distinct"] == 4096
    assert k[5]["trunc_min"] == k[5]["trunc_max"] == 0x3F800000
    assert not (k[6]["single_value"] or k[6]["frequent"] or k[6]["structured"] or k[6]["approx"])
    # PC7: (e mod 10 + 1)/10; slice start 458752 = 2 mod 10 -> residues 2..7 get 6554
    cnt = {r: (6554 if 2 <= r <= 7 else 6553) for r in range(10)}
    tenths = [f32((r + 1) / 10) for r in range(10)]
    order = sorted(range(10), key=lambda r: (-cnt[r], tenths[r]))[:8]
    assert k[7]["n_distinct"] == 10 and k[7]["heavy"] == 255 and k[7]["dict8"]
    assert list(k[7]["top_bits"][:8]) == [tenths[r] for r in order]
    assert list(k[7]["top_count"][:8]) == [cnt[r] for r in order]
    assert k[8]["n_st_eq_pre"] == 65536 and k[8]["single_zero"]                  # P1/P2
    assert k[9]["n_st_eq_pre"] == 32768
    assert k[10]["structured"] and k[10]["p_x"] == CFG1_BASE + 4 * 655360
    assert O.y_of(k[10]["q_ylo"], k[10]["q_yhi"]) == 11 * 65536 - 1
    # PC11: zero unless e mod 250 == 0 over [720896, 786432): 262 multiples of 250
    assert k[11]["n_zero"] == 65274 and k[11]["n_st_eq_pre"] == 65274 and k[11]["frequent"]
    assert not k[11]["single_zero"] and k[11]["top_count"][0] == 65274
    assert not (k[12]["single_value"] or k[12]["frequent"] or k[12]["structured"])
    assert k[13]["n_zero"] == 32768 and k[13]["n_distinct"] == 2 and k[13]["n_st_eq_pre"] == 32768   # Q8
    assert list(k[13]["top_bits"][:2]) == [0, 0x80000000]
    assert k[14]["heavy"] == 0 and k[14]["dict8"] and k[14]["n_distinct"] == 256
    assert k[15]["heavy"] == 8                                                  # k/64, |k|<=1024 -> f16


def test_cfg1_snapshot_diff(cfg1):
    cfg, objs, recs, keys, glob, objstat = cfg1
    d = O.snapshot_diff(cfg, objs, recs, 0, O.DIFF_WRITTEN)
    assert d["n_masked"] == 524288
    assert d["n_unchanged"] == 65536 + 32768 + 65274 + 32768 == 196346
    assert d["n_changed"] == 524288 - 196346 and d["n_untouched"] == 0 and d["redundant"] == 1  # 37.45% > 33%
    d = O.snapshot_diff(cfg, objs, recs, 0, O.DIFF_ALL)
    assert d["n_masked"] == 1 << 20 and d["n_unchanged"] == 196346 + 524288      # load slices unchanged


# --------------------------------------------------------------------------
# The paper's worked examples P1-P14
# --------------------------------------------------------------------------

def test_p1_figure3_program():
    """P:L263 Figure 3: memset(A,0), memset(B,0); kernel stores 0 to A; line 7 reads A."""
    n = 1000
    A, B = 0x100000, 0x200000
    objs = [obj(A, 4 * n, 0, 4, zeros(4 * n), zeros(4 * n)), obj(B, 4 * n, 1, 4, zeros(4 * n), zeros(4 * n))]
    rows = [(A + 4 * i, 0, 0, meta(4, S, 1)) for i in range(n)]          # line 5: store 0 to A
    rows += [(A + 4 * i, 0, 1, meta(4, S, 0)) for i in range(n)]         # line 7: read A
    rows += [(B + 4 * i, 0, 2, meta(4, S, 1)) for i in range(n)]         # line 7: write B
    recs = records(rows)
    cfg = O.make_config(3)
    keys, glob, objstat = O.analyze(cfg, objs, recs)
    assert keys[0]["n_st_eq_pre"] == n and keys[0]["single_zero"]
    assert keys[1]["n_ld_eq_pre"] == n and keys[1]["single_zero"]
    d = O.snapshot_diff(cfg, objs, recs, 0)
    assert (d["n_masked"], d["n_unchanged"], d["redundant"]) == (n, n, 1)


def _darknet(M=4, K=6, N=10, T=4):
    """P:L54-L76 Listing 1: fill_ongpu zeroes output, then gemm(beta=1) loads and stores C."""
    WA, WB, WC = 0x10000000, 0x20000000, 0x30000000
    a_vals = [f32(0.5 + i) for i in range(M * K)]
    b_vals = [f32(-1.0 - i) for i in range(K * N)]
    c_vals = [f32(7.0 + i) for i in range(M * N)]
    pre_c = zeros(4 * M * N)
    post_c = le_bytes(c_vals, 4)
    objs = [obj(WA, 4 * M * K, 0, 4, le_bytes(a_vals, 4), le_bytes(a_vals, 4)),
            obj(WB, 4 * K * N, 1, 4, le_bytes(b_vals, 4), le_bytes(b_vals, 4)),
            obj(WC, 4 * M * N, 2, 4, pre_c, post_c)]
    fill = [(WC + 4 * i, 0, 0, meta(4, F, 1)) for i in range(M * N)]
    gemm = []
    for mt in range(0, M, T):
        for nt in range(0, N, T):
            for k in range(K):
                for m in range(mt, min(mt + T, M)):
                    gemm.append((WA + 4 * (m * K + k), a_vals[m * K + k], 1, meta(4, F)))
                for nn in range(nt, min(nt + T, N)):
                    gemm.append((WB + 4 * (k * N + nn), b_vals[k * N + nn], 2, meta(4, F)))
            for m in range(mt, min(mt + T, M)):
                for nn in range(nt, min(nt + T, N)):
                    gemm.append((WC + 4 * (m * N + nn), 0, 3, meta(4, F)))
                    gemm.append((WC + 4 * (m * N + nn), c_vals[m * N + nn], 4, meta(4, F, 1)))
    return objs, records(fill), records(gemm)


def test_p2_darknet_fill_then_gemm():
    M, K, N, T = 4, 6, 10, 4
    objs, fill, gemm = _darknet(M, K, N, T)
    cfg = O.make_config(5)
    fill_objs = [dict(o) for o in objs]
    fill_objs[2] = dict(objs[2], post=zeros(4 * M * N))                # after fill_ongpu: zeros
    keys, _, _ = O.analyze(cfg, fill_objs, fill)
    assert keys[0]["n_st_eq_pre"] == keys[0]["n_st"] == M * N and keys[0]["single_zero"]
    d = O.snapshot_diff(cfg, fill_objs, fill, 2)
    assert d["n_unchanged"] == d["n_masked"] == M * N and d["redundant"]  # 100% unchanged
    keys, _, objstat = O.analyze(cfg, objs, gemm)
    n_ntiles, n_mtiles = -(-N // T), -(-M // T)
    assert keys[3]["single_zero"] and keys[3]["n_ld_eq_pre"] == keys[3]["n_ld"] == M * N   # redundant zero loads
    assert keys[4]["n_st_eq_pre"] == 0
    assert objstat[0]["n_ld_reload"] == (n_ntiles - 1) * M * K             # A re-read per N tile
    assert objstat[1]["n_ld_reload"] == (n_mtiles - 1) * K * N


def test_p3_darknet_duplicate_copy():
    """P:L66-L76 Listing 2: output_gpu and x_gpu are copies of the same zeroed l.output."""
    n = 4096
    flip = zeros(n)
    flip[1234] = 1
    objs = [obj(0x1000000, n, 0, 4, None, zeros(n)), obj(0x2000000, n, 1, 4, None, zeros(n)),
            obj(0x3000000, n, 2, 4, None, flip), obj(0x4000000, n // 2, 3, 4, None, zeros(n // 2)),
            obj(0x5000000, n, 4, 4, None, None)]
    assert list(O.object_dedup(objs)) == [0, 0, 2, 3, 4]


def test_p4_lavamd_tenths():
    """rA holds ten values {0.1..1.0} -> n_distinct 10, dict8, not a narrower type."""
    counts = [5, 3, 8, 1, 9, 2, 7, 4, 6, 10]
    rows, i = [], 0
    for k, c in enumerate(counts):
        for _ in range(c):
            rows.append((0x1000 + 8 * i, f64((k + 1) / 10), 0, meta(8, F)))
            i += 1
    cfg = O.make_config(1)
    keys, _, _ = O.analyze(cfg, [], records(rows))
    k = keys[0]
    order = sorted(range(10), key=lambda j: -counts[j])[:8]
    assert k["n_distinct"] == 10 and k["dict8"] and k["heavy"] == 255
    assert list(k["top_count"][:8]) == [counts[j] for j in order]
    assert list(k["top_bits"][:8]) == [f64((j + 1) / 10) for j in order]
    # equal counts: ties break by bits ascending (Q18)
    rows = [(0x1000 + 8 * i, f64((i % 10 + 1) / 10), 0, meta(8, F)) for i in range(100)]
    keys, _, _ = O.analyze(cfg, [], records(rows))
    assert list(keys[0]["top_bits"][:8]) == sorted(f64((j + 1) / 10) for j in range(10))[:8]


@pytest.mark.parametrize("kind,w,vals,heavy", [
    (S, 4, range(-1, 101), 4),                   # bfs g_cost int32 -> int8
    (U, 4, range(0, 256), 0),
    (U, 4, range(0, 257), 1),
    (S, 2, range(-129, 6), 255),
    (S, 8, [-(1 << 31), (1 << 31) - 1], 6),
    (S, 8, [-(1 << 31) - 1, 0], 255),
    (U, 8, [0, (1 << 32) - 1], 2),
    (U, 1, [0, 255], 255),
])
def test_p5_heavy_type_integer(kind, w, vals, heavy):
    mask = (1 << (8 * w)) - 1
    rows = [(0x1000 + w * i, v & mask, 0, meta(w, kind)) for i, v in enumerate(vals)]
    keys, _, _ = O.analyze(O.make_config(1), [], records(rows))
    assert keys[0]["heavy"] == heavy


def test_p6_barracuda_zeros():
    """99.6% zeros in global_alns -> frequent 0, not single zero."""
    rows = [(0x1000 + 4 * i, 0 if i % 250 else f32(1.0 + i), 0, meta(4, F, 1)) for i in range(1000)]
    keys, _, _ = O.analyze(O.make_config(1), [], records(rows))
    k = keys[0]
    assert (k["top_bits"][0], k["top_count"][0]) == (0, 996) and k["frequent"] and not k["single_zero"]


def test_p7_hotspot3d_approx():
    """tIn_d single-valued within 2% -> K=7 truncation single value (Q6)."""
    rows = [(0x1000 + 4 * i, 0x3F800000 + (i * 37 % (1 << 14)), 0, meta(4, F)) for i in range(500)]
    keys, _, _ = O.analyze(O.make_config(1), [], records(rows))
    assert keys[0]["approx"] and not keys[0]["single_value"]
    rows = [(0x1000 + 4 * i, f32(0.999 if i % 2 else 1.001), 0, meta(4, F)) for i in range(500)]
    keys, _, _ = O.analyze(O.make_config(1), [], records(rows))
    assert not keys[0]["approx"]                                   # straddles a truncation bucket


def test_p8_srad_structured():
    """srad_v1 d_iN[i] = i-1 is linear in the address; the clamped iN[0]=0 is not."""
    n, base = 512, 0x5000
    rows = [(base + 4 * i, (i - 1) & 0xFFFFFFFF, 0, meta(4, S)) for i in range(1, n)]
    keys, _, _ = O.analyze(O.make_config(1), [], records(rows))
    k = keys[0]
    assert k["structured"] and (k["p_x"], O.y_of(k["p_ylo"], k["p_yhi"])) == (base + 4, 0)
    assert (k["q_x"], O.y_of(k["q_ylo"], k["q_yhi"])) == (base + 4 * (n - 1), n - 2)
    keys, _, _ = O.analyze(O.make_config(1), [], records(rows + [(base, 0, 0, meta(4, S))]))
    assert keys[0]["line_state"] == O.LINE_FAIL and not keys[0]["structured"]


def test_p9_resnet_ones():
    """the ones tensor -> single value; 1.0f fits u8."""
    rows = [(0x1000 + 4 * i, f32(1.0), 0, meta(4, F)) for i in range(300)]
    keys, _, _ = O.analyze(O.make_config(1), [], records(rows))
    assert keys[0]["single_value"] and keys[0]["heavy"] == 0 and not keys[0]["approx"]


def test_p10_deepwave_zero_twice():
    """zeros_like then zero_(): the second zero-fill rewrites zeros."""
    n = 777
    objs = [obj(0x9000, 4 * n, 0, 4, zeros(4 * n), zeros(4 * n))]
    recs = records((0x9000 + 4 * i, 0, 0, meta(4, F, 1)) for i in range(n))
    cfg = O.make_config(1)
    keys, _, _ = O.analyze(cfg, objs, recs)
    assert keys[0]["n_st_eq_pre"] == keys[0]["n_st"] == n and keys[0]["single_zero"]
    d = O.snapshot_diff(cfg, objs, recs, 0)
    assert d["n_unchanged"] == d["n_masked"] == n and d["redundant"]


def test_p11_castro_a_is_one():
    """a == 1.0 mostly; the slope store then rewrites the pre value."""
    npt = 2000
    A, SL = 0x100000, 0x200000
    a_vals = [f64(1.0) if p % 20 else f64(0.5 + p) for p in range(npt)]
    s_pre = [f64(3.0 + p) for p in range(npt)]
    s_new = [s_pre[p] if p % 20 else f64(-1.0 - p) for p in range(npt)]
    objs = [obj(A, 8 * npt, 0, 8, le_bytes(a_vals, 8), le_bytes(a_vals, 8)),
            obj(SL, 8 * npt, 1, 8, le_bytes(s_pre, 8), le_bytes(s_new, 8))]
    rows = []
    for p in range(npt):
        rows.append((A + 8 * p, a_vals[p], 0, meta(8, F)))
        rows.append((SL + 8 * p, s_new[p], 1, meta(8, F, 1)))
    keys, _, _ = O.analyze(O.make_config(2), objs, records(rows))
    assert (keys[0]["top_bits"][0], keys[0]["top_count"][0]) == (0x3FF0000000000000, 1900)
    assert keys[1]["n_st_eq_pre"] == 1900


def test_p12_backprop_zero_objects():
    """w and oldw are all zeros -> single zero per object."""
    n = 300
    objs = [obj(0x10000, 8 * n, 0, 8, zeros(8 * n), zeros(8 * n)), obj(0x20000, 8 * n, 1, 8, zeros(8 * n), zeros(8 * n))]
    rows = [(0x10000 + 8 * i, 0, 0, meta(8, F)) for i in range(n)] + \
           [(0x20000 + 8 * i, 0, 1, meta(8, F)) for i in range(n)]
    keys, _, _ = O.analyze(O.make_config(2), objs, records(rows))
    assert keys[2]["single_zero"] and keys[3]["single_zero"]          # object keys n_pcs + id


def test_p13_huffman_histo():
    """most values written to histo are zeros -> frequent values."""
    rows = [(0x1000 + 4 * (i % 256), 0 if i % 10 else i + 1, 0, meta(4, U, 1)) for i in range(1000)]
    keys, _, _ = O.analyze(O.make_config(1), [], records(rows))
    assert keys[0]["frequent"] and (keys[0]["top_bits"][0], keys[0]["top_count"][0]) == (0, 900)


def test_p14_bert_padding_rows():
    """masked_fill_ re-zeroes padding rows already zero -> redundant stores = padding elements."""
    R, D, pad_rows = 16, 24, [0, 5, 11]
    pre = [0 if r in pad_rows else f32(1.0 + r * D + d) for r in range(R) for d in range(D)]
    objs = [obj(0x40000, 4 * R * D, 0, 4, le_bytes(pre, 4), le_bytes(pre, 4))]
    rows = [(0x40000 + 4 * (r * D + d), 0, 0, meta(4, F, 1)) for r in pad_rows for d in range(D)]
    keys, _, _ = O.analyze(O.make_config(1), objs, records(rows))
    assert keys[0]["n_st_eq_pre"] == len(pad_rows) * D


# --------------------------------------------------------------------------
# Validity, mapping and snapshot edge cases (SURVEY 8(b) errors; Q20, Q21)
# --------------------------------------------------------------------------

def test_invalid_unmapped_shared_straddle():
    base = 0x10000
    pre = le_bytes(range(16), 4)
    objs = [obj(base, 64, 0, 4, pre, pre)]
    rows = [
        (base, 0, 0, meta(4, U) | (1 << 7)),            # reserved meta bit -> invalid
        (base, 0, 0, meta(1, F)),                       # float of width 1 -> invalid
        (base, 0, 0, meta(4, BF)),                      # bf16 of width 4 -> invalid
        (base, 0, 9, meta(4, U)),                       # pc >= n_pcs -> invalid
        (base, 1 << 32, 0, meta(4, U)),                 # bits above 8w -> invalid
        (1 << 48, 0, 0, meta(4, U)),                    # addr >= 2^48 -> invalid
        (base + 64, 0, 0, meta(4, U)),                  # unmapped (just past the end)
        (base + 62, 0x0F, 0, meta(4, U)),               # straddles the end: maps, no snapshot (Q21)
        (base + 4, 1, 0, meta(4, U)),                   # eq_pre
        (base + 5, 0x02000000, 0, meta(4, U)),          # misaligned, eq_pre bytewise: bytes 5..8 = 0,0,0,2
        (100, 7, 0, meta(4, U, 0, 1)),                  # shared space (Q20)
    ]
    keys, glob, objstat = O.analyze(O.make_config(2), objs, records(rows))
    assert glob["n_invalid"] == 6 and glob["n_unmapped"] == 1
    assert keys[0]["n_ld"] == 5 and keys[0]["n_ld_eq_pre"] == 2 and keys[0]["n_nosnap"] == 3
    assert keys[2]["n_ld"] == 3 and keys[2]["n_nosnap"] == 1                 # object key
    assert keys[3]["n_ld"] == 1 and keys[3]["n_nosnap"] == 1                 # SHARED key
    assert objstat[0]["n_loaded_eq"] == 1 and objstat[0]["n_ld_reload"] == 1     # both start in element 1


def test_written_bitmap_wide_store_and_partial_elem():
    base = 0x20000
    pre = zeros(10)
    objs = [obj(base, 10, 0, 4, pre, le_bytes([1, 0, 0], 4)[:10])]       # 3 elements, last one 2 bytes
    rows = [(base, 0, 0, meta(8, U, 1)), (base + 8, 0, 0, meta(2, U, 1))]
    cfg = O.make_config(1)
    d = O.snapshot_diff(cfg, objs, records(rows), 0)
    assert (d["n_elems"], d["n_masked"], d["n_unchanged"], d["n_untouched"]) == (3, 3, 2, 0)
    d = O.snapshot_diff(cfg, objs, records(rows), 0, O.DIFF_MASK, np.array([0b101], dtype=np.uint32))
    assert (d["n_masked"], d["n_unchanged"]) == (2, 1)


# --------------------------------------------------------------------------
# Bit-level helpers against independent library routines
# --------------------------------------------------------------------------

def _np_flags(vals64, is_f64):
    import torch
    v = vals64
    nan = np.isnan(v)
    with np.errstate(invalid="ignore", over="ignore"):
        nonint = nan | np.isinf(v) | (np.trunc(np.where(np.isfinite(v), v, 0)) != v) | \
            ((v == 0) & np.signbit(v)) | (np.abs(v) >= 2.0 ** 63)
        nf16 = nan | (v.astype(np.float16).astype(np.float64) != v)
        nbf16 = nan | (torch.from_numpy(v).to(torch.bfloat16).to(torch.float64).numpy() != v)
        nf32 = (nan | (v.astype(np.float32).astype(np.float64) != v)) if is_f64 else np.zeros_like(nan)
    return nan | (nonint << 1) | (nf16 << 2) | (nbf16 << 3) | (nf32 << 4)


def test_float_flags_exhaustive_16bit():
    bits = np.arange(65536, dtype=np.uint64)
    h = bits.astype(np.uint16).view(np.float16).astype(np.float64)
    exp = _np_flags(h, False)
    got = np.array([O.float_flags(int(b), F, 2) for b in bits], dtype=np.int64)
    assert np.array_equal(got, exp)
    bf = (bits.astype(np.uint32) << 16).view(np.float32).astype(np.float64)
    exp = _np_flags(bf, False)
    got = np.array([O.float_flags(int(b), BF, 2) for b in bits], dtype=np.int64)
    assert np.array_equal(got, exp)


def test_float_flags_random_32_64():
    rng = np.random.default_rng(5)
    b32 = rng.integers(0, 1 << 32, 20000, dtype=np.uint64)
    edge32 = [f32(x) for x in (0.0, -0.0, 1.0, 65504.0, 65520.0, 2.0 ** -24, 2.0 ** -25, 3.0 * 2 ** -26,
                               float("inf"), 2.0 ** 63, -(2.0 ** 63), 1.5, 255.0, 16777216.0)]
    b32 = np.concatenate([b32, np.array(edge32 + [0x7FC00001, 0xFF800000], dtype=np.uint64)])
    exp = _np_flags(b32.astype(np.uint32).view(np.float32).astype(np.float64), False)
    got = np.array([O.float_flags(int(b), F, 4) for b in b32], dtype=np.int64)
    assert np.array_equal(got, exp)
    b64 = rng.integers(0, 1 << 63, 20000, dtype=np.uint64) * np.uint64(2) + rng.integers(0, 2, 20000, dtype=np.uint64)
    small = np.array([f64(x) for x in rng.integers(-3000, 3000, 2000) / 8.0], dtype=np.uint64)
    b64 = np.concatenate([b64, small, np.array([f64(x) for x in (1e300, 2.0 ** 63, 0.1, 3.0)], dtype=np.uint64)])
    exp = _np_flags(b64.view(np.float64), True)
    got = np.array([O.float_flags(int(b), F, 8) for b in b64], dtype=np.int64)
    assert np.array_equal(got, exp)


@pytest.mark.parametrize("kind,w", [(U, 1), (U, 2), (U, 4), (U, 8), (S, 1), (S, 2), (S, 4), (S, 8), (F, 2),
                                    (F, 4), (F, 8), (BF, 2)])
def test_ord_orders_like_the_numbers(kind, w):
    """C5: sorting by ord equals sorting by numeric value (-0.0 just below +0.0), NaNs aside."""
    rng = np.random.default_rng(kind * 16 + w)
    vals = [int(x) for x in rng.integers(0, 1 << (8 * w) if w < 8 else (1 << 63), 3000, dtype=np.uint64)]
    vals += [0, (1 << (8 * w)) - 1, 1 << (8 * w - 1)]

    def num(b):
        if kind == U:
            return (b, 0)
        if kind == S:
            return (b - (1 << (8 * w)) if b >> (8 * w - 1) else b, 0)
        if kind == BF:
            v = float(np.array([b << 16], dtype=np.uint32).view(np.float32)[0])
        else:
            dt = {2: np.float16, 4: np.float32, 8: np.float64}[w]
            it = {2: np.uint16, 4: np.uint32, 8: np.uint64}[w]
            v = float(np.array([b], dtype=it).view(dt)[0])
        if v != v:
            return None
        return (v, 0 if (v == 0 and b >> (8 * w - 1)) else 1)

    pairs = [(num(b), O.ord_key(b, kind, w)) for b in vals if num(b) is not None]
    by_num = sorted(pairs, key=lambda p: p[0])
    ords = [p[1] for p in by_num]
    assert ords == sorted(ords)


def test_trunc_closed_forms():
    assert O.trunc(0x3F80FFFF, F, 4, 7) == 0x3F800000
    assert O.trunc(0x3F81FFFF, F, 4, 7) == 0x3F810000
    assert O.trunc(0x3FF0123456789ABC, F, 8, 7) == 0x3FF0000000000000
    assert O.trunc(0x3C07, F, 2, 7) == 0x3C00 and O.trunc(0x3C0F, F, 2, 7) == 0x3C08
    assert O.trunc(0x3F85, BF, 2, 7) == 0x3F85 and O.trunc(0x3F85, BF, 2, 3) == 0x3F80


# --------------------------------------------------------------------------
# Brute force on tiny random traces + invariants
# --------------------------------------------------------------------------

POOL = {1: [0, 1, 7, 0x80, 0xFF], 2: [0, 1, 0x3C00, 0x8000, 0x7E00, 0x3F80, 0xFFFF, 0x4500],
        4: [0, 1, 0x2A, 0x3F800000, 0x80000000, 0x7FC00000, 0xFFFFFFFF, 0x42280000, 0x40A00000],
        8: [0, 1, 0x3FF0000000000000, 0x8000000000000000, 0xFFFFFFFFFFFFFFFF, 0x4014000000000000,
            0x7FF8000000000000, 0x3FB999999999999A]}
COMBOS = [(U, 1), (U, 2), (U, 4), (U, 8), (S, 1), (S, 2), (S, 4), (S, 8), (F, 2), (F, 4), (F, 8), (BF, 2)]


def _tiny(seed, n=1500, structured_pc=None):
    rng = np.random.default_rng(seed)
    o0 = rng.integers(0, 256, 256, dtype=np.uint8)
    o0_post = o0.copy()
    o0_post[rng.integers(0, 256, 40)] ^= 1
    objs = [obj(0x1000, 256, 0, 4, o0, o0_post), obj(0x2000, 100, 1, 2, zeros(100), None)]
    rows = []
    for i in range(n):
        pc = int(rng.integers(0, 8))
        kind, w = COMBOS[int(rng.integers(0, len(COMBOS)))] if pc != structured_pc else (S, 4)
        a = int(rng.choice([0x1000 + rng.integers(0, 260), 0x2000 + rng.integers(0, 104), 0x3000]))
        shared = int(rng.random() < 0.1)
        if pc == structured_pc:
            a = 0x1000 + 4 * int(rng.integers(0, 64))
            v = ((a - 0x1000) // 4 * 5 - 9) & 0xFFFFFFFF
            shared = 0
        else:
            v = POOL[w][int(rng.integers(0, len(POOL[w])))]
        rows.append((a, v, pc, meta(w, kind, int(rng.integers(0, 2)), shared)))
    return objs, records(rows)


def _key_members(recs, objs, n_pcs):
    """record indices per key (brute force mapping, valid records only)"""
    members = {}
    for i, r in enumerate(recs):
        m = int(r["meta"])
        w, kind = 1 << (m & 3), (m >> 2) & 3
        if (m >> 6) or (kind == F and w == 1) or (kind == BF and w != 2) or r["pc"] >= n_pcs or \
                int(r["addr"]) >= 1 << 48:
            continue
        if w < 8 and int(r["value"]) >> (8 * w):
            continue
        members.setdefault(int(r["pc"]), []).append(i)
        if (m >> 5) & 1:
            members.setdefault(n_pcs + len(objs), []).append(i)
            continue
        for o in objs:
            if o["base"] <= int(r["addr"]) < o["base"] + o["size"]:
                members.setdefault(n_pcs + o["id"], []).append(i)
    return members


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_brute_force_histogram_topk(seed):
    """B1: O(n^2) pair counting gives every count; top-k by (count desc, bits asc)."""
    objs, recs = _tiny(seed)
    cfg = O.make_config(8, topk=4)
    keys, glob, _ = O.analyze(cfg, objs, recs)
    for key, idx in _key_members(recs, objs, 8).items():
        vals = [int(recs[i]["value"]) for i in idx]
        counts = {}
        for a in vals:
            counts[a] = sum(1 for b in vals if b == a)
        top = sorted(counts.items(), key=lambda kv: (-kv[1], kv[0]))[:4]
        k = keys[key]
        assert k["n_distinct"] == len(counts)
        assert [(int(b), int(c)) for b, c in zip(k["top_bits"][:k["n_top"]], k["top_count"][:k["n_top"]])] == top
        assert k["n_ld"] + k["n_st"] == len(vals)
        assert k["raw_min"] == min(vals) and k["raw_max"] == max(vals)


@pytest.mark.parametrize("seed", [4, 5])
def test_brute_force_structured(seed):
    """B2: LINE iff some pair's line passes through every point (and one y per x)."""
    objs, recs = _tiny(seed, n=300, structured_pc=3)
    keys, _, _ = O.analyze(O.make_config(8), objs, recs)
    for key, idx in _key_members(recs, objs, 8).items():
        pts = []
        fail = False
        for i in idx:
            m = int(recs[i]["meta"])
            w, kind = 1 << (m & 3), (m >> 2) & 3
            b = int(recs[i]["value"])
            if kind == U:
                y = b
            elif kind == S:
                y = b - (1 << (8 * w)) if b >> (8 * w - 1) else b
            else:
                fl = O.float_flags(b, kind, w)
                if fl & 2:
                    fail = True
                    break
                if kind == BF:
                    y = int(np.array([b << 16], dtype=np.uint32).view(np.float32)[0])
                else:
                    dt = {2: np.float16, 4: np.float32, 8: np.float64}[w]
                    it = {2: np.uint16, 4: np.uint32, 8: np.uint64}[w]
                    y = int(np.array([b], dtype=it).view(dt)[0])
            pts.append((int(recs[i]["addr"]), y))
        if fail:
            assert keys[key]["line_state"] == O.LINE_FAIL
            continue
        pts = sorted(set(pts))
        xs = {x for x, _ in pts}
        if len(xs) < len(pts):
            exp = O.LINE_FAIL
        elif len(pts) == 1:
            exp = O.LINE_POINT
        else:
            exp = O.LINE_FAIL
            for a in pts:
                for b in pts:
                    if a[0] < b[0] and all((y - a[1]) * (b[0] - a[0]) == (b[1] - a[1]) * (x - a[0]) for x, y in pts):
                        exp = O.LINE_LINE
        assert keys[key]["line_state"] == exp, key
        if exp == O.LINE_LINE:
            assert (keys[key]["p_x"], O.y_of(keys[key]["p_ylo"], keys[key]["p_yhi"])) == pts[0]
            assert (keys[key]["q_x"], O.y_of(keys[key]["q_ylo"], keys[key]["q_yhi"])) == pts[-1]
    assert keys[3]["structured"] == 1


def test_brute_force_dedup():
    """B3 / I9: pairwise byte comparison; classes named by their min id."""
    rng = np.random.default_rng(9)
    base = [rng.integers(0, 256, 64, dtype=np.uint8) for _ in range(4)]
    objs = []
    for i in range(40):
        c = int(rng.integers(0, 6))
        data = base[c % 4].copy() if c < 4 else zeros(64) if c == 4 else rng.integers(0, 256, 64, dtype=np.uint8)
        if rng.random() < 0.1:
            data[int(rng.integers(0, 64))] ^= 0x40
        size = 64 if rng.random() < 0.9 else 32
        objs.append(obj(0x100000 * (i + 1), size, int(rng.permutation(40)[0]) if False else i, 8, None,
                        data if rng.random() > 0.05 else None))
    g = O.object_dedup(objs)
    for i, a in enumerate(objs):
        exp = i
        if a["post"] is not None:
            for j, b in enumerate(objs):
                if b["post"] is not None and b["size"] == a["size"] and \
                        bytes(a["post"][:a["size"]]) == bytes(b["post"][:b["size"]]):
                    exp = min(exp, j)
        assert g[i] == exp
        assert g[g[i]] == g[i]                                   # I9: class representative is itself


def _candidates(kind, w):
    out = []
    for v in (1, 2, 4):
        if v >= w:
            break
        out.append(("int", v))
        if kind in (F, BF) and v == 2:
            out += [("f16", 2), ("bf16", 2)]
        if kind in (F, BF) and v == 4:
            out.append(("f32", 4))
    return out


def test_brute_force_heavy_type():
    """B4: enumerate candidate types in increasing width and convert every value."""
    import torch
    rng = np.random.default_rng(11)
    cases = [(F, 4, [f32(x) for x in (1.0, 2.0, 255.0)]), (F, 4, [f32(x) for x in (-3.0, 100.0)]),
             (F, 8, [f64(x) for x in (0.5, 1.25)]), (F, 8, [f64(x) for x in (70000.0, 1.0)]),
             (F, 8, [f64(x) for x in (3.0e38, 1.0)]), (F, 4, [f32(x) for x in (-0.0, 1.0)]),
             (BF, 2, [0x3F80, 0x4300]), (BF, 2, [0x3F81, 0x4049]), (F, 2, [0x3C00, 0x3C01]),
             (F, 8, [f64(x) for x in (65504.0, -2.0)]), (F, 4, [f32(x) for x in (70000.0, 3.5)])]
    for _ in range(30):
        kind, w = [(F, 4), (F, 8), (BF, 2), (F, 2)][int(rng.integers(0, 4))]
        scale = float(2.0 ** int(rng.integers(-3, 20)))
        vals = [float(x) for x in np.round(rng.normal(0, scale, 5) * 4) / 4]
        bits = {4: lambda x: f32(x), 8: lambda x: f64(x)}
        if kind == F and w in bits:
            cases.append((kind, w, [bits[w](x) for x in vals]))
    for kind, w, bl in cases:
        rows = [(0x1000 + w * i, b, 0, meta(w, kind)) for i, b in enumerate(bl)]
        keys, _, _ = O.analyze(O.make_config(1), [], records(rows))
        if kind == BF:
            vals = [float(np.array([b << 16], dtype=np.uint32).view(np.float32)[0]) for b in bl]
        else:
            dt = {2: np.float16, 4: np.float32, 8: np.float64}[w]
            it = {2: np.uint16, 4: np.uint32, 8: np.uint64}[w]
            vals = [float(np.array([b], dtype=it).view(dt)[0]) for b in bl]
        exp = 255
        for cand, v in _candidates(kind, w):
            if cand == "int":
                if all(x == int(x) and not (x == 0 and np.signbit(x)) for x in vals):
                    if min(vals) >= 0 and max(vals) <= 2 ** (8 * v) - 1:
                        exp = {1: 0, 2: 1, 4: 2}[v]
                    elif min(vals) < 0 and min(vals) >= -2 ** (8 * v - 1) and max(vals) <= 2 ** (8 * v - 1) - 1:
                        exp = {1: 4, 2: 5, 4: 6}[v]
            elif cand == "f16":
                if all(float(np.float16(x)) == x for x in vals):
                    exp = 8
            elif cand == "bf16":
                if all(float(torch.tensor(x, dtype=torch.float64).to(torch.bfloat16)) == x for x in vals):
                    exp = 11
            elif cand == "f32":
                if all(float(np.float32(x)) == x for x in vals):
                    exp = 9
            if exp != 255:
                break
        assert keys[0]["heavy"] == exp, (kind, w, vals)


@pytest.mark.parametrize("seed", [21, 22])
def test_invariants_on_fuzz(seed):
    """I1-I8 and I10 (permutation invariance) on the adversarial generator."""
    n = 20000
    objs = G.objects(G.FUZZ)
    full = [dict(o, pre=G.snapshot_host(G.FUZZ, 0, seed, i, 0) if o["has_pre"] else None,
                 post=G.snapshot_host(G.FUZZ, 0, seed, i, 1) if o["has_post"] else None) for i, o in enumerate(objs)]
    recs = G.records_host(G.FUZZ, 0, seed, 0, n)
    cfg = O.make_config(64)
    keys, glob, objstat = O.analyze(cfg, full, recs)
    npc, nob = 64, len(objs)
    tot = lambda k: int(k["n_ld"]) + int(k["n_st"])
    assert sum(tot(k) for k in keys[:npc]) == n - glob["n_invalid"]                                 # I1
    shared = keys[npc + nob]
    assert glob["n_invalid"] > 0 and glob["n_unmapped"] > 0 and tot(shared) > 0
    valid_global = sum(tot(k) for k in keys[:npc]) - tot(shared)
    assert sum(tot(k) for k in keys[npc:npc + nob]) + glob["n_unmapped"] == valid_global              # I2
    for k in keys:                                                                                  # I3, I6
        assert k["n_zero"] <= tot(k) and k["n_ld_eq_pre"] <= k["n_ld"] and k["n_st_eq_pre"] <= k["n_st"]
        c = list(k["top_count"][:k["n_top"]])
        assert c == sorted(c, reverse=True) and sum(c) <= tot(k) and k["n_top"] == min(8, k["n_distinct"])
        if k["single_value"]:                                                                       # I5
            assert k["n_distinct"] == 1 and k["top_bits"][0] == k["raw_min"] and k["top_count"][0] == tot(k)
    for s in objstat:
        assert 0 <= s["n_ld_reload"] and s["n_loaded_eq"] <= s["n_elems"]
    members = _key_members(recs, full, npc)
    for key, idx in members.items():                                                                # I4
        v = recs["value"][idx]
        assert keys[key]["raw_min"] == v.min() and keys[key]["raw_max"] == v.max()
    assert any(k["line_state"] == O.LINE_LINE for k in keys[:npc])                                  # I7 exercised
    for i, o in enumerate(full):                                                                    # I8
        if o["pre"] is not None and o["post"] is not None:
            d = O.snapshot_diff(cfg, full, recs, i, O.DIFF_ALL)
            assert d["n_unchanged"] + d["n_changed"] == d["n_masked"] == d["n_elems"]
    perm = np.random.default_rng(seed).permutation(n)                                               # I10
    k2, g2, o2 = O.analyze(cfg, full, recs[perm])
    assert k2.tobytes() == keys.tobytes() and g2.tobytes() == glob.tobytes() and o2.tobytes() == objstat.tobytes()
