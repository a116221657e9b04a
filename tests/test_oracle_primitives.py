"""Pins of the CPU oracle's primitives against things other than itself (not gpu).

Each test names what fixes the expected value: an RFC known-answer vector, Python big-integer
arithmetic, a closed form of PAPER.md Sec. 2.2, or an exhaustive enumeration of a toy ring.
"""
import numpy as np
import pytest

from oracle import bruteforce as bf

SEED = 0x50534D4C


# --- ChaCha20: RFC 8439 known-answer vectors (R1) ----------------------------------
def test_chacha20_rfc8439_sec_2_3_2(orc):
    key = np.frombuffer(bytes(range(32)), dtype="<u4")
    nonce = np.frombuffer(bytes.fromhex("000000090000004a00000000"), dtype="<u4")
    out = orc.chacha20_block(key, 1, nonce)
    expect = bytes.fromhex(
        "10f1e7e4d13b5915500fdd1fa32071c4c7d1f4c733c068030422aa9ac3d46c4e"
        "d2826446079faa0914c2d705d98b02a2b5129cd1de164eb9cbd083e8a2503c4e")
    assert out.astype("<u4").tobytes() == expect


def test_chacha20_rfc8439_appendix_a1_zero_key(orc):
    out = orc.chacha20_block(np.zeros(8, np.uint32), 0, np.zeros(3, np.uint32))
    expect = bytes.fromhex(
        "76b8e0ada0f13d90405d6ae55386bd28bdd219b8a08ded1aa836efcc8b770dc7"
        "da41597c5157488d7724e03fb8d84a376a43b8f41518a11cc387b669b2ee6586")
    assert out.astype("<u4").tobytes() == expect


def test_prg_stream_layout(orc):
    """Element e of a stream = little-endian word pair (l=64) / word (l=32) of block e/8 (e/16)."""
    seed, call = 0x0123456789ABCDEF, 0x1122334455667788
    t = orc.tag("U0")
    key = np.array([seed & 0xFFFFFFFF, seed >> 32, 0, 0, 0, 0, 0, 0], np.uint32)
    nonce = np.array([t, call & 0xFFFFFFFF, call >> 32], np.uint32)
    v64 = orc.prg(64, seed, t, call, 40)
    v32 = orc.prg(32, seed, t, call, 40)
    for e in range(40):
        blk = orc.chacha20_block(key, e // 8, nonce).astype(np.uint64)
        j = e % 8
        assert int(v64[e]) == int(blk[2 * j]) | (int(blk[2 * j + 1]) << 32)
        blk = orc.chacha20_block(key, e // 16, nonce)
        assert int(v32[e]) == int(blk[e % 16])
    # offsets address the same stream
    assert np.array_equal(orc.prg(64, seed, t, call, 13, offset=27), v64[27:40])
    # uniformity sanity: mean of 2^16 l=64 words close to 2^63
    v = orc.prg(64, SEED, orc.tag("SH"), 7, 1 << 16).astype(np.float64)
    assert abs(v.mean() / 2.0 ** 63 - 1.0) < 0.02


# --- fixed-point encoding (R3) -------------------------------------------------------
def test_encode_round_half_even_and_decode(orc):
    f = 13
    xs = [0.0, 0.5 / 2 ** f, 1.5 / 2 ** f, 2.5 / 2 ** f, -0.5 / 2 ** f, -1.5 / 2 ** f, 1.0, -1.0,
          0.123456789, -3.75, 1000.0009765625]
    v = orc.encode(np.array(xs), 64, f)
    for x, got in zip(xs, v):
        want = round(x * 2 ** f) % (1 << 64)  # Python round() is round-half-to-even
        assert int(got) == want
    back = orc.decode(v, 64, f)
    assert np.all(np.abs(back - np.array(xs)) <= 2.0 ** -(f + 1))
    v32 = orc.encode(np.array([-1.0, 2.0]), 32, f)
    assert [int(t) for t in v32] == [(1 << 32) - (1 << 13), 1 << 14]
    assert list(orc.decode(v32, 32, f)) == [-1.0, 2.0]


# --- sharing --------------------------------------------------------------
@pytest.mark.parametrize("l", [8, 16, 32, 64])
def test_share_reconstructs(orc, l):
    rng = np.random.default_rng(1)
    x = rng.integers(0, 2 ** min(l, 63), 1000, dtype=np.uint64)
    x0, x1 = orc.share(x, SEED + 1, 5, l)
    assert np.array_equal(x0, orc.prg(l, SEED + 1, orc.tag("SH"), 5, 1000))
    for a, b, c in zip(x0[:50], x1[:50], x[:50]):
        assert (int(a) + int(b)) % (1 << l) == int(c)
    assert np.array_equal(orc.reconstruct(x0, x1, l), x)


# --- ring matmul vs Python big integers ---------------------------------------------------------
@pytest.mark.parametrize("l", [8, 16, 32, 64])
@pytest.mark.parametrize("shape", [(4, 4, 4), (3, 5, 2), (7, 1, 9), (1, 13, 1)])
def test_ring_matmul_bruteforce(orc, l, shape):
    M, K, N = shape
    A = orc.prg(l, SEED, orc.tag("tA"), M * 100 + K, M * K).reshape(M, K)
    B = orc.prg(l, SEED, orc.tag("tB"), K * 100 + N, K * N).reshape(K, N)
    C = orc.ring_matmul(A, B, l)
    assert bf.to_int_matrix(C) == bf.matmul_mod(bf.to_int_matrix(A), bf.to_int_matrix(B), l)


def test_ring_matmul_worst_case_all_ones(orc):
    """All-ones operands: C = K * (2^64 - 1)^2 mod 2^64 = K mod 2^64 (closed form)."""
    K = 300
    A = np.full((3, K), 0xFFFFFFFFFFFFFFFF, np.uint64)
    B = np.full((K, 2), 0xFFFFFFFFFFFFFFFF, np.uint64)
    assert np.all(orc.ring_matmul(A, B) == K)


# --- triplets (Eqs. 2-3) --------------------------------------------------------------
@pytest.mark.parametrize("l", [16, 32, 64])
def test_triplet_validity(orc, l):
    M, K, N = 4, 5, 3
    U0, U1, V0, V1, Z0, Z1 = orc.triplet_gen(SEED + 2, 99, M, K, N, l)
    U = bf.add_mod(U0, U1, l)
    V = bf.add_mod(V0, V1, l)
    assert bf.add_mod(Z0, Z1, l) == bf.matmul_mod(U, V, l)
    # each party's own streams come from its own seed s_i = PRG(dealer seed, "KD", i) (R4, R23):
    # U0 / V0 / Z0 from s_0, U1 / V1 from s_1; only Z1 needs both
    s0, s1 = orc.party_seed(SEED + 2, 0), orc.party_seed(SEED + 2, 1)
    assert s0 != s1 and SEED + 2 not in (s0, s1)
    assert s0 == int(orc.prg(64, SEED + 2, orc.tag("KD"), 0, 1)[0])
    assert np.array_equal(U0.reshape(-1), orc.prg(l, s0, orc.tag("U0"), 99, M * K))
    assert np.array_equal(Z0.reshape(-1), orc.prg(l, s0, orc.tag("Z0"), 99, M * N))
    assert np.array_equal(V1.reshape(-1), orc.prg(l, s1, orc.tag("V1"), 99, K * N))
    h = orc.hadamard_triplet_gen(SEED + 2, 100, 50, l)
    for t in range(50):
        u = int(h[0][t]) + int(h[1][t])
        v = int(h[2][t]) + int(h[3][t])
        assert (int(h[4][t]) + int(h[5][t])) % (1 << l) == (u * v) % (1 << l)


# --- Beaver matmul (Eqs. 4-8) --------------------------------------------------------
@pytest.mark.parametrize("l", [8, 32, 64])
@pytest.mark.parametrize("shape", [(4, 4, 4), (3, 5, 2), (6, 1, 7)])
def test_beaver_matmul_reconstructs_and_matches_bruteforce(orc, l, shape):
    M, K, N = shape
    A = orc.prg(l, SEED, orc.tag("tA"), 1, M * K).reshape(M, K)
    B = orc.prg(l, SEED, orc.tag("tB"), 2, K * N).reshape(K, N)
    A0, A1 = orc.share(A, SEED + 1, 10, l)
    B0, B1 = orc.share(B, SEED + 1, 11, l)
    trip = orc.triplet_gen(SEED + 2, 12, M, K, N, l)
    AB = bf.matmul_mod(bf.to_int_matrix(A), bf.to_int_matrix(B), l)
    (C0, C1), tr = orc.beaver_matmul((A0, A1), (B0, B1), trip, l=l, trace=True)
    assert bf.add_mod(C0, C1, l) == AB                                   # Eq. 1 reconstructed
    E = bf.add_mod(A, bf.add_mod(trip[0], trip[1], l), l, sign=-1)      # E = A - U
    F = bf.add_mod(B, bf.add_mod(trip[2], trip[3], l), l, sign=-1)
    assert bf.to_int_matrix(tr["E"]) == E and bf.to_int_matrix(tr["F"]) == F
    assert bf.to_int_matrix(tr["E0"]) == bf.add_mod(A0, trip[0], l, sign=-1)
    for i in range(2):
        want = bf.beaver_shares_bj(E, F, trip[i], trip[2 + i], trip[4 + i], i, l)
        assert bf.to_int_matrix((C0, C1)[i]) == want
    # the paper's Eq. 6 form: different shares, same reconstruction; equals Eq. 8 per party
    P0, P1 = orc.beaver_matmul((A0, A1), (B0, B1), trip, form=1, l=l)
    assert bf.add_mod(P0, P1, l) == AB
    for i, (Ai, Bi, Pi) in enumerate(((A0, B0, P0), (A1, B1, P1))):
        assert bf.to_int_matrix(Pi) == bf.beaver_eq8(E, F, Ai, Bi, trip[4 + i], i, l)
        assert bf.to_int_matrix(Pi) == bf.beaver_shares_paper(E, F, Ai, Bi, trip[4 + i], i, l)


def test_beaver_hadamard_reconstructs(orc):
    n, l = 500, 64
    a = orc.prg(l, SEED, orc.tag("ha"), 0, n)
    b = orc.prg(l, SEED, orc.tag("hb"), 0, n)
    A = orc.share(a, SEED + 1, 1, l)
    B = orc.share(b, SEED + 1, 2, l)
    C0, C1 = orc.beaver_hadamard(A, B, orc.hadamard_triplet_gen(SEED + 2, 3, n, l), l)
    for t in range(n):
        assert (int(C0[t]) + int(C1[t])) % 2 ** 64 == (int(a[t]) * int(b[t])) % 2 ** 64


# --- truncation (SecureML Thm. 1, restated in BASELINE north_star) -----------------------------
@pytest.mark.parametrize("l,d,lx", [(64, 13, 40), (32, 13, 18), (64, 14, 30)])
def test_truncation_secureml_bound(orc, l, d, lx):
    """|t - floor(x/2^d)| <= 1 except w.p. <= 2^(lx+1-l); both outcomes are floor or floor+1."""
    n = 200000
    rng = np.random.default_rng(l * 100 + d)
    xs = rng.integers(-(2 ** lx), 2 ** lx, n, dtype=np.int64)
    x = (xs.astype(np.uint64)) & orc.mask(l)
    x0, x1 = orc.share(x, SEED + 1, 77 + d, l)
    t = orc.reconstruct(orc.truncate(x0, 0, d, l), orc.truncate(x1, 1, d, l), l)
    tv = np.array([bf.signed(v, l) for v in t], dtype=np.int64)
    fl = xs >> d
    diff = tv - fl
    bad = np.count_nonzero((diff != 0) & (diff != 1))
    assert bad <= max(3, int(8 * n * 2.0 ** (lx + 1 - l)))
    # stochastic rounding: P(+1) = frac(x / 2^d) (R7); compare the means
    frac = (xs - (fl << d)) / 2.0 ** d
    ok = (diff == 0) | (diff == 1)
    assert abs(diff[ok].mean() - frac[ok].mean()) < 0.01


def test_truncation_special_cases(orc):
    x = np.array([0, 1, 8191, 8192, 123456789, 2 ** 40], np.uint64)
    # c1 = 0 and x >= 0: exact floor; d = 0: identity
    assert np.array_equal(orc.truncate(x, 0, 13), x >> np.uint64(13))
    assert np.array_equal(orc.truncate(np.zeros(6, np.uint64), 1, 13), np.zeros(6, np.uint64))
    assert np.array_equal(orc.truncate(x, 1, 0), x)
    for c in [0, 1, 5, 2 ** 63, 2 ** 64 - 1, 2 ** 64 - 8192]:
        got = int(orc.truncate(np.array([c], np.uint64), 1, 13)[0])
        assert got == (-((-c % 2 ** 64) >> 13)) % 2 ** 64  # party 1 = -floor(-c / 2^d)


# --- MSB / DReLU / ReLU / Eq. 9: exhaustive over toy rings ------------------------------------
@pytest.mark.parametrize("l,splits", [(8, 8), (16, 1)])
def test_secure_msb_exhaustive(orc, l, splits):
    n = 1 << l
    x = np.arange(n, dtype=np.uint64)
    for s in range(splits):
        x0, x1 = orc.share(x, SEED + 1, 1000 + s, l)
        mat = orc.msb_dealer(SEED + 2, 2000 + s, n, l)
        (a0, a1), (b0, b1) = orc.secure_msb((x0, x1), mat, l, want_bool=True)
        want = (x >> np.uint64(l - 1)) & np.uint64(1)
        assert np.array_equal(b0 ^ b1, want)
        assert np.array_equal((a0 + a1) & orc.mask(l), want)


def test_secure_msb_l64_edges(orc):
    l = 64
    vals = [0, 1, 2 ** 63 - 1, 2 ** 63, 2 ** 64 - 1, 4096, 2 ** 64 - 4096, 2 ** 62, 3 * 2 ** 62]
    rng = np.random.default_rng(5)
    vals += [int(v) for v in rng.integers(0, 2 ** 63, 2000, dtype=np.uint64)]
    vals += [int(v) + 2 ** 63 for v in rng.integers(0, 2 ** 63, 2000, dtype=np.uint64)]
    x = np.array(vals, dtype=np.uint64)
    x0, x1 = orc.share(x, SEED + 1, 3, l)
    mat = orc.msb_dealer(SEED + 2, 4, x.size, l)
    a0, a1 = orc.secure_msb((x0, x1), mat, l)
    assert [int(v) for v in orc.reconstruct(a0, a1)] == [bf.msb(v, 64) for v in vals]


@pytest.mark.parametrize("l,gates", [(64, 182), (32, 87), (16, 40), (8, 17)])
def test_reduced_msb_material_layout(orc, l, gates):
    """R27: 11 material words per element and party; the AND material occupies exactly the gate
    bits of the reduced prefix (l = 64: 63 + 2*31 + 31 + 15 + 7 + 3 + 1 = 182 of 12 x 64 full-word
    AND bits), nothing outside them, and every group is a valid boolean triplet."""
    n = 4096
    assert orc.lib().or_msb_material_words(l, n) == 11 * n
    m0, m1 = orc.msb_dealer(SEED + 2, 77, n, l)
    union = 0
    for g in range(3):
        a = m0[(3 * g) * n:(3 * g + 1) * n] ^ m1[(3 * g) * n:(3 * g + 1) * n]
        b = m0[(3 * g + 1) * n:(3 * g + 2) * n] ^ m1[(3 * g + 1) * n:(3 * g + 2) * n]
        c = m0[(3 * g + 2) * n:(3 * g + 3) * n] ^ m1[(3 * g + 2) * n:(3 * g + 3) * n]
        assert np.array_equal(c, a & b)
        seen = 0
        for w in (a, b, m0[(3 * g) * n:(3 * g + 1) * n]):
            for v in w.tolist():
                seen |= v
        union += bin(seen).count("1")
    assert union == gates   # 4096 random words light up every gate bit and nothing else
    assert set(np.unique(m0[9 * n:10 * n]).tolist()) <= {0, 1}


def test_secure_relu_and_eq9_exhaustive_l16(orc):
    l, f = 16, 4
    n = 1 << l
    x = np.arange(n, dtype=np.uint64)
    X = orc.share(x, SEED + 1, 31, l)
    (r0, r1), (d0, d1) = orc.secure_relu(X, orc.msb_dealer(SEED + 2, 32, n, l),
                                         orc.hadamard_triplet_gen(SEED + 2, 33, n, l), l)
    r = orc.reconstruct(r0, r1, l)
    d = orc.reconstruct(d0, d1, l)
    assert [int(v) for v in r] == [bf.relu_fixed(v, l) % (1 << l) for v in range(n)]
    assert [int(v) for v in d] == [1 - bf.msb(v, l) for v in range(n)]
    y0, y1 = orc.secure_eq9(X, orc.msb_dealer(SEED + 2, 34, 2 * n, l),
                            orc.hadamard_triplet_gen(SEED + 2, 35, 2 * n, l), l, f)
    y = orc.reconstruct(y0, y1, l)
    # Eq. 9 on the grid; x +- 1/2 must not wrap, so compare where |x| < 2^(l-1) - 2^(f-1)
    lim = (1 << (l - 1)) - (1 << (f - 1))
    for v in range(n):
        if abs(bf.signed(v, l)) < lim:
            assert int(y[v]) == bf.eq9_fixed(v, l, f), v


# --- CSR delta codec --------------------------------------------------------
def test_csr_delta_codec(orc):
    rng = np.random.default_rng(9)
    prev = rng.integers(0, 2 ** 63, (16, 20), dtype=np.uint64)
    cur = prev.copy()
    idx = rng.choice(320, 80, replace=False)          # exactly 25% changed -> CSR (>= 75% zeros)
    cur.reshape(-1)[idx] += np.uint64(12345)
    enc = orc.delta_csr_encode(cur, prev)
    assert enc["is_csr"] and enc["nnz"] == 80
    assert np.array_equal(orc.delta_csr_apply(prev, enc), cur)
    cur.reshape(-1)[rng.choice(np.setdiff1d(np.arange(320), idx), 1)] += np.uint64(1)
    enc = orc.delta_csr_encode(cur, prev)             # 81 nonzeros -> dense
    assert not enc["is_csr"]
    assert np.array_equal(orc.delta_csr_apply(prev, enc), cur)
    enc = orc.delta_csr_encode(prev, prev)            # persistent mask, constant data: empty CSR
    assert enc["is_csr"] and enc["nnz"] == 0 and np.array_equal(orc.delta_csr_apply(prev, enc), prev)


def test_dealer_key_separation(orc):
    """DESIGN.md R23: every material stream of party i is keyed by s_i alone; the dealer-only FSS
    mask stream and the derived words are not reproducible from either party seed."""
    seed = 0x1234
    s0, s1 = orc.party_seed(seed, 0), orc.party_seed(seed, 1)
    for t, want in (("U0", s0), ("V0", s0), ("Z0", s0), ("RA", s0), ("FS", s0), ("F0", s0), ("K0", s0),
                    ("U1", s1), ("V1", s1), ("R1", s1), ("K1", s1), ("FR", seed)):
        assert orc.stream_seed(seed, orc.tag(t)) == want, t
    for t in range(12):   # boolean AND triplet streams a_i^t, b_i^t, c_0^t
        assert orc.stream_seed(seed, orc.tag(bytes([ord("a"), ord("0"), t]))) == s0
        assert orc.stream_seed(seed, orc.tag(bytes([ord("b"), ord("1"), t]))) == s1
        assert orc.stream_seed(seed, orc.tag(bytes([ord("c"), ord("0"), t]))) == s0
    m0, m1 = orc.msb_dealer(seed, 5, 64)
    n = 64
    # party 1's a/b words from s_1 alone (masked to the round-0 gate bits 0..62, R27); its c words
    # are derived (need a_0, b_0 too)
    mask0 = np.uint64((1 << 63) - 1)
    assert np.array_equal(m1[:n], orc.prg(64, s1, orc.tag(bytes([ord("a"), ord("1"), 0])), 5, n) & mask0)
    assert not np.array_equal(m1[2 * n:3 * n], orc.prg(64, s1, orc.tag(bytes([ord("c"), ord("1"), 0])), 5, n))
