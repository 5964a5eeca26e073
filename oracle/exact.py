"""Exact-rational single-tile Winograd F(2x2,3x3) -- TEST INFRASTRUCTURE ONLY.

Pure-Python ``fractions.Fraction`` arithmetic for one 4x4 input tile d and one
3x3 filter g, written from Yan, Wang & Chu (PPoPP'20), /root/reference/PAPER.md:

* Eq. 1 (L85):  O = A^T [ (G g G^T) (.) (B^T d B) ] A
* Eq. 2-3 (L89-113): A^T, G, B^T (garbled in the scrape; reconstructed as the
  Lavin-Gray matrices -- DESIGN.md readings R1/R2) -- pinned by the identity
  tests in tests/test_oracle.py, not by re-typing.
* L115: FTF needs 28 float instructions, ITF 32 float additions, OTF 24 float
  additions -- pinned by ``count_*`` below against tests/golden/paper_constants.json.

Only tests/ import this module.  It shares nothing with the CUDA path.
"""
from __future__ import annotations

from fractions import Fraction as Fr

AT = [[Fr(1), Fr(1), Fr(1), Fr(0)],
      [Fr(0), Fr(1), Fr(-1), Fr(-1)]]
G = [[Fr(1), Fr(0), Fr(0)],
     [Fr(1, 2), Fr(1, 2), Fr(1, 2)],
     [Fr(1, 2), Fr(-1, 2), Fr(1, 2)],
     [Fr(0), Fr(0), Fr(1)]]
BT = [[Fr(1), Fr(0), Fr(-1), Fr(0)],
      [Fr(0), Fr(1), Fr(1), Fr(0)],
      [Fr(0), Fr(-1), Fr(1), Fr(0)],
      [Fr(0), Fr(1), Fr(0), Fr(-1)]]


def transpose(m):
    return [list(r) for r in zip(*m)]


def matmul(a, b):
    return [[sum((a[i][t] * b[t][j] for t in range(len(b))), Fr(0))
             for j in range(len(b[0]))] for i in range(len(a))]


def ftf(g):
    """Eq. 5 (L191): U = G g G^T for a 3x3 filter g (lists of Fractions)."""
    return matmul(matmul(G, g), transpose(G))


def itf(d):
    """Eq. 6 (L193-195): V = B^T d B for a 4x4 input tile d."""
    return matmul(matmul(BT, d), transpose(BT))


def ewmm(u, v):
    """Eq. 7 (L197-203) for a single channel: element-wise product U (.) V."""
    return [[u[i][j] * v[i][j] for j in range(4)] for i in range(4)]


def otf(m):
    """Eq. 8 (L205-207): Y = A^T M A for a 4x4 pre-transform tile."""
    return matmul(matmul(AT, m), transpose(AT))


def winograd_tile(d, g):
    """Eq. 1 (L85): the 2x2 output of F(2x2,3x3) for one tile/filter pair."""
    return otf(ewmm(ftf(g), itf(d)))


def _nonzero_pattern(m):
    return [[x != 0 for x in row] for row in m]


def count_adds_linear_map(m):
    """Additions needed to apply a {0,+-1}-coefficient matrix m to one vector:
    sum over rows of (nonzeros - 1).  Used for the ITF/OTF counts of L115."""
    return sum(max(0, sum(1 for x in row if x != 0) - 1) for row in m)


def count_itf_adds():
    """B^T d B: B^T applied to the 4 columns of d, then B^T to the 4 rows of (B^T d)."""
    return 4 * count_adds_linear_map(BT) + 4 * count_adds_linear_map(BT)


def count_otf_adds():
    """A^T M A: A^T applied to the 4 columns of M, then to the 2 rows of (A^T M)."""
    return 4 * count_adds_linear_map(AT) + 2 * count_adds_linear_map(AT)


class _Counted:
    """A Fraction that counts the float instructions (FADD / FMUL / FFMA) spent on it."""
    ops = 0

    def __init__(self, v):
        self.v = Fr(v)

    def __add__(self, o):
        _Counted.ops += 1
        return _Counted(self.v + o.v)

    def __sub__(self, o):
        _Counted.ops += 1
        return _Counted(self.v - o.v)

    def scale(self, k):  # FMUL by a constant
        _Counted.ops += 1
        return _Counted(k * self.v)

    def fma(self, k, c):  # FFMA: k * self + c in one instruction
        _Counted.ops += 1
        return _Counted(k * self.v + c.v)


def _g_vector_schedule(a, b, c):
    """G applied to one 3-vector (a, b, c) with the cheapest schedule G's structure allows: rows 0 and 3
    of G copy a and c (0 instructions); rows 1 and 2 are 0.5 (a + c) +- 0.5 b = h +- 0.5 b with
    h = 0.5 (a + c): FADD, FMUL, 2 FFMA."""
    h = (a + c).scale(Fr(1, 2))
    return [a, b.fma(Fr(1, 2), h), b.fma(Fr(-1, 2), h), c]


def ftf_counted(g):
    """G g G^T (Eq. 5) through _g_vector_schedule on the 3 columns of g, then on the 4 rows of G g;
    returns (u as Fractions, float instructions used)."""
    _Counted.ops = 0
    gc = [[_Counted(g[r][s]) for s in range(3)] for r in range(3)]
    cols = [_g_vector_schedule(gc[0][s], gc[1][s], gc[2][s]) for s in range(3)]  # (G g)[:, s]
    t = [[cols[s][r] for s in range(3)] for r in range(4)]                          # G g, 4 x 3
    u = [_g_vector_schedule(*t[r]) for r in range(4)]                                # (G g) G^T
    return [[u[r][s].v for s in range(4)] for r in range(4)], _Counted.ops


def count_ftf_instructions():
    """Float instructions of the FTF (L115 prints 28): counted by executing the schedule on a tile and
    checking that the schedule really computes G g G^T (an exact product with G from Eq. 3), so that a
    wrong or more expensive schedule fails the pin."""
    g = [[Fr(3, 7), Fr(-2), Fr(5, 3)], [Fr(1, 9), Fr(4), Fr(-6, 5)], [Fr(7), Fr(-1, 4), Fr(2, 11)]]
    u, ops = ftf_counted(g)
    assert u == ftf(g), "counted FTF schedule does not compute G g G^T"
    return ops


def correlate_tile(d, g):
    """Brute force: 2x2 valid correlation of a 4x4 tile with a 3x3 filter (no flip)."""
    return [[sum((d[y + r][x + s] * g[r][s] for r in range(3) for s in range(3)), Fr(0))
             for x in range(2)] for y in range(2)]


def convolve_tile_flipped(d, g):
    """2x2 valid *convolution* (flipped filter) -- used to show the orientation."""
    return [[sum((d[y + r][x + s] * g[2 - r][2 - s] for r in range(3) for s in range(3)), Fr(0))
             for x in range(2)] for y in range(2)]


# --------------------------------------------------------------------------
# NEXT row N1: F(4x4,3x3) (Lavin-Gray matrices, points 0, +-1, +-2, inf).
# PAPER.md gives no F(4x4) matrices (it cites [11, 26], L117); these are pinned
# only by the exact identity below (tests/test_oracle.py).
# --------------------------------------------------------------------------
AT4 = [[Fr(v) for v in row] for row in [[1, 1, 1, 1, 1, 0], [0, 1, -1, 2, -2, 0], [0, 1, 1, 4, 4, 0],
                                         [0, 1, -1, 8, -8, 1]]]
G4 = [[Fr(1, 4), Fr(0), Fr(0)],
      [Fr(-1, 6), Fr(-1, 6), Fr(-1, 6)],
      [Fr(-1, 6), Fr(1, 6), Fr(-1, 6)],
      [Fr(1, 24), Fr(1, 12), Fr(1, 6)],
      [Fr(1, 24), Fr(-1, 12), Fr(1, 6)],
      [Fr(0), Fr(0), Fr(1)]]
BT4 = [[Fr(v) for v in row] for row in [[4, 0, -5, 0, 1, 0], [0, -4, -4, 1, 1, 0], [0, 4, -4, -1, 1, 0],
                                         [0, -2, -1, 2, 1, 0], [0, 2, -1, -2, 1, 0], [0, 4, 0, -5, 0, 1]]]


def winograd_f4_tile(d, g):
    """F(4x4,3x3): AT4 [(G4 g G4^T) (.) (BT4 d BT4^T)] AT4^T for a 6x6 tile d, 3x3 filter g."""
    u = matmul(matmul(G4, g), transpose(G4))
    v = matmul(matmul(BT4, d), transpose(BT4))
    m = [[u[i][j] * v[i][j] for j in range(6)] for i in range(6)]
    return matmul(matmul(AT4, m), transpose(AT4))


def correlate_tile_f4(d, g):
    """Brute force: 4x4 valid correlation of a 6x6 tile with a 3x3 filter."""
    return [[sum((d[y + r][x + s] * g[r][s] for r in range(3) for s in range(3)), Fr(0))
             for x in range(4)] for y in range(4)]
