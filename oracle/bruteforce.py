"""Pure-Python big-integer definitions for tiny inputs -- TEST INFRASTRUCTURE ONLY.

These are the independent pins of the C oracle: arbitrary-precision integer arithmetic reduced
mod 2^l only at the end, written from the mathematical definitions (no uint64 wraparound, no
shared code with psml_oracle.c).  Sizes: a few elements to a few hundred.
"""


def to_int_matrix(a):
    return [[int(v) for v in row] for row in a]


def matmul_mod(A, B, l):
    """(A . B) mod 2^l over the integers, then reduced (Eq. 1 in Z_{2^l})."""
    M, K, N = len(A), len(B), len(B[0])
    mod = 1 << l
    return [[sum(int(A[i][k]) * int(B[k][j]) for k in range(K)) % mod for j in range(N)]
            for i in range(M)]


def add_mod(A, B, l, sign=1):
    mod = 1 << l
    return [[(int(a) + sign * int(b)) % mod for a, b in zip(ra, rb)] for ra, rb in zip(A, B)]


def signed(v, l):
    v = int(v) % (1 << l)
    return v - (1 << l) if v >> (l - 1) else v


def msb(v, l):
    return (int(v) >> (l - 1)) & 1


def floor_div_pow2(x_signed, d):
    """floor(x / 2^d) for a signed integer (Python >> is floor division for negatives)."""
    return x_signed >> d


def relu_fixed(v, l):
    s = signed(v, l)
    return s if s >= 0 else 0


def eq9_fixed(v, l, f):
    """PAPER.md Eq. 9 on the fixed-point grid: 0 below -1/2, x + 1/2 between, 1 above."""
    s = signed(v, l)
    half, one = 1 << (f - 1), 1 << f
    if s < -half:
        return 0
    if s > half:
        return one
    return s + half


def beaver_shares_bj(E, F, U_i, V_i, Z_i, i, l):
    """C_i = i.E.F + E.V_i + U_i.F + Z_i (BASELINE north_star form) with big ints."""
    EF = matmul_mod(E, F, l)
    EV = matmul_mod(E, V_i, l)
    UF = matmul_mod(U_i, F, l)
    mod = 1 << l
    return [[(i * EF[r][c] + EV[r][c] + UF[r][c] + int(Z_i[r][c])) % mod
             for c in range(len(Z_i[0]))] for r in range(len(Z_i))]


def beaver_shares_paper(E, F, A_i, B_i, Z_i, i, l):
    """C_i = (-i) x E x F + A_i x F + E x B_i + Z_i (Eq. 6) with big ints."""
    EF = matmul_mod(E, F, l)
    AF = matmul_mod(A_i, F, l)
    EB = matmul_mod(E, B_i, l)
    mod = 1 << l
    return [[(-i * EF[r][c] + AF[r][c] + EB[r][c] + int(Z_i[r][c])) % mod
             for c in range(len(Z_i[0]))] for r in range(len(Z_i))]


def beaver_eq8(E, F, A_i, B_i, Z_i, i, l):
    """PAPER.md Eq. 8 (L175): ((-i) E + A_i | E) x (F ; B_i) + Z_i, one K-concatenated GEMM."""
    mod = 1 << l
    M, K = len(E), len(E[0])
    left = [[(-i * int(E[r][k]) + int(A_i[r][k])) % mod for k in range(K)] + [int(e) for e in E[r]]
            for r in range(M)]
    right = [[int(v) for v in row] for row in F] + [[int(v) for v in row] for row in B_i]
    P = matmul_mod(left, right, l)
    return [[(P[r][c] + int(Z_i[r][c])) % mod for c in range(len(Z_i[0]))] for r in range(M)]


def truncate_share(c, party, d, l):
    """SecureML local truncation with big ints: party 0 floor(c/2^d); party 1 -floor(-c/2^d)."""
    mod = 1 << l
    c = int(c) % mod
    if party == 0:
        return c >> d
    return (-(((-c) % mod) >> d)) % mod
