#!/usr/bin/env python3
"""Hand derivation, in exact rational arithmetic, of the conv3d worked rounding examples
(tests/golden/conv3d_worked_examples.txt).

Independent of oracle/ and of the CUDA path: only `fractions.Fraction` and the IEEE-754 rule
"round to nearest, ties to even" written out below (rn). It evaluates DESIGN.md reading C1 — the
PolyBench/GPU conv3D body the paper benchmarks (§V.B) — at the centre of a
3x3x3 grid, every product and every partial sum rounded to the array type, terms added left to right
in Polybench's order, and records every intermediate value so the file can be checked by eye.

It also evaluates plausible WRONG readings of the same body (other summation orders, FMA
contraction, merged coefficients, per-plane grouping) and only accepts an input whose correct result
differs from every one of them, so the golden bits pin the order and the absence of contraction.

Inputs: A(dk,dj,di) = rn(x / M) with M = 2^61 - 1 and x the Lehmer sequence x <- 48271 x mod M
started at seed * 0x9E3779B97F4A7C15 mod M (27 values, dk slowest, di fastest). A single example cannot tell
every wrong reading apart, so examples are taken for seeds 1, 2, 3, ... and kept while they catch a
wrong reading no kept example catches yet, until every wrong reading is caught by at least one
example (a deterministic greedy cover; the seeds are written into the file).

usage: python tests/golden/derive_conv3d_worked.py > tests/golden/conv3d_worked_examples.txt
"""
from fractions import Fraction as F

# (mantissa bits incl. hidden, min normal exponent) per type
FMT = {"f64": (53, -1022), "f32": (24, -126)}

# reading C1: Polybench's 15 terms in its order, (coefficient, dk, dj, di); Polybench's outer index
# is our plane index k, its inner index is our contiguous i
TERMS = [(2, -1, -1, -1), (4, 1, -1, -1), (5, -1, -1, -1), (7, 1, -1, -1), (-8, -1, -1, -1),
         (10, 1, -1, -1), (-3, 0, -1, 0), (6, 0, 0, 0), (-9, 0, 1, 0), (2, -1, -1, 1),
         (4, 1, -1, 1), (5, -1, 0, 1), (7, 1, 0, 1), (-8, -1, 1, 1), (10, 1, 1, 1)]


def rn(x, fmt):
    """Round the rational x to the nearest value of the binary format, ties to even (normal range)."""
    if x == 0:
        return F(0)
    p, emin = FMT[fmt]
    s = -1 if x < 0 else 1
    a = abs(x)
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if F(2) ** e > a:
        e -= 1
    while F(2) ** (e + 1) <= a:
        e += 1
    assert e >= emin, "subnormal range not needed here"
    ulp = F(2) ** (e - p + 1)
    q = a / ulp
    n = q.numerator // q.denominator
    rem = q - n
    if rem > F(1, 2) or (rem == F(1, 2) and n % 2 == 1):
        n += 1
    return s * n * ulp


def bits(x, fmt):
    """IEEE bit pattern of a value already representable in fmt (normal or zero)."""
    p, emin = FMT[fmt]
    ebits, width = (11, 64) if fmt == "f64" else (8, 32)
    if x == 0:
        return 0
    s = 1 if x < 0 else 0
    a = abs(x)
    e = a.numerator.bit_length() - a.denominator.bit_length()
    if F(2) ** e > a:
        e -= 1
    while F(2) ** (e + 1) <= a:
        e += 1
    m = a / F(2) ** (e - p + 1)
    assert m.denominator == 1, "not representable"
    frac = int(m) - (1 << (p - 1))
    bias = (1 << (ebits - 1)) - 1
    return (s << (width - 1)) | ((e + bias) << (p - 1)) | frac


def hx(x, fmt):
    return ("0x%016x" if fmt == "f64" else "0x%08x") % bits(x, fmt)


M61 = (1 << 61) - 1


def lehmer(seed, n):
    x, out = (seed * 0x9E3779B97F4A7C15) % M61, []   # spread small seeds over [1, M)
    for _ in range(n):
        x = (48271 * x) % M61
        out.append(x)
    return out


def inputs(seed, fmt):
    xs = iter(lehmer(seed, 27))
    return {(dk, dj, di): rn(F(next(xs), M61), fmt)
            for dk in (-1, 0, 1) for dj in (-1, 0, 1) for di in (-1, 0, 1)}


def left_to_right(A, terms, fmt, fma=False, trace=None):
    s = None
    for c, dk, dj, di in terms:
        a = A[(dk, dj, di)]
        if fma and s is not None:
            s = rn(F(c) * a + s, fmt)           # fused: one rounding of c*a + s
            if trace is not None:
                trace.append((c, dk, dj, di, F(c) * a, None, s))
            continue
        t = rn(F(c) * a, fmt)
        new = t if s is None else rn(s + t, fmt)
        if trace is not None:
            trace.append((c, dk, dj, di, F(c) * a, t, new))
        s = new
    return s


def tree(vals, fmt):
    while len(vals) > 1:
        nxt = [rn(vals[i] + vals[i + 1], fmt) for i in range(0, len(vals) - 1, 2)]
        if len(vals) % 2:
            nxt.append(vals[-1])
        vals = nxt
    return vals[0]


def alternatives(A, fmt):
    """Plausible wrong readings of the same body; each must give different bits."""
    alt = {}
    alt["reversed_order"] = left_to_right(A, TERMS[::-1], fmt)
    alt["fma_contracted"] = left_to_right(A, TERMS, fmt, fma=True)
    for i in range(1, len(TERMS) - 1):          # swapping terms 0 and 1 is commutative: skipped
        t = list(TERMS)
        t[i], t[i + 1] = t[i + 1], t[i]
        alt[f"swap_terms_{i}_{i + 1}"] = left_to_right(A, t, fmt)
    # coefficients of repeated offsets merged first (sum c exactly, one product per distinct operand)
    merged = {}
    for c, dk, dj, di in TERMS:
        merged[(dk, dj, di)] = merged.get((dk, dj, di), 0) + c
    alt["merged_coefficients"] = left_to_right(A, [(c,) + k for k, c in merged.items()], fmt)
    # grouped by plane: the dk = -1, 0, +1 partial sums, then added
    parts = [left_to_right(A, [t for t in TERMS if t[1] == g], fmt) for g in (-1, 0, 1)]
    alt["per_plane_groups"] = rn(rn(parts[0] + parts[1], fmt) + parts[2], fmt)
    alt["pairwise_tree"] = tree([rn(F(c) * A[(dk, dj, di)], fmt) for c, dk, dj, di in TERMS], fmt)
    # operands transposed: Polybench's outer index taken as our contiguous i (dk <-> di)
    alt["dk_di_transposed"] = left_to_right(A, [(c, di, dj, dk) for c, dk, dj, di in TERMS], fmt)
    return alt


def main():
    out = []
    w = out.append
    w("# Worked rounding examples for the 3-D convolution body (PAPER.md §V.B, P:L606-638, names Polybench")
    w("# 3DCONV but prints no formula; DESIGN.md reading C1 takes the PolyBench/GPU conv3D body).")
    w("# Derived by tests/golden/derive_conv3d_worked.py in exact rational arithmetic (fractions.Fraction,")
    w("# round-to-nearest-even written out), independent of oracle/ and of the CUDA path.")
    w("# Each example is the centre of a 3x3x3 grid; inputs are rn(x/(2^61-1)) of a Lehmer sequence (see the script).")
    w("# Every product c*A and every partial sum is rounded to the array type; terms are added left to right")
    w("# in Polybench's order; no FMA. `step` lines: coefficient, offset, exact product, rounded product,")
    w("# rounded running sum. `alt` lines: the result of a WRONG reading (other summation order, FMA")
    w("# contraction, merged coefficients, grouping, transposed operands) where it differs from `result`;")
    w("# every wrong reading differs in at least one example, so the result bits pin the order and the")
    w("# absence of contraction.")
    for fmt in ("f64", "f32"):
        kept, caught = [], set()
        names = list(alternatives(inputs(1, fmt), fmt))
        for seed in range(1, 5000):
            A = inputs(seed, fmt)
            r = left_to_right(A, TERMS, fmt)
            alt = alternatives(A, fmt)
            new = {k for k, v in alt.items() if bits(v, fmt) != bits(r, fmt)} - caught
            if new:
                kept.append(seed)
                caught |= new
            if len(caught) == len(names):
                break
        else:
            raise SystemExit(f"no cover for {fmt}: missing {set(names) - caught}")
        for seed in kept:
            A = inputs(seed, fmt)
            w(f"example {fmt} seed {seed}")
            for dk in (-1, 0, 1):
                for dj in (-1, 0, 1):
                    for di in (-1, 0, 1):
                        w(f"input {fmt} {seed} {dk:+d} {dj:+d} {di:+d} {hx(A[(dk, dj, di)], fmt)}  # {float(A[(dk, dj, di)])!r}")
            trace = []
            r = left_to_right(A, TERMS, fmt, trace=trace)
            for n, (c, dk, dj, di, exact, t, s) in enumerate(trace):
                w(f"step {fmt} {seed} {n:2d} c={c:+d} ({dk:+d},{dj:+d},{di:+d}) product={float(exact)!r} "
                  f"rn(product)={hx(t, fmt)} sum={hx(s, fmt)} ({float(s)!r})")
            w(f"result {fmt} {seed} {hx(r, fmt)}  # {float(r)!r}")
            exact = sum(F(c) * A[(dk, dj, di)] for c, dk, dj, di in TERMS)
            w(f"# exact rational value of the 15 terms: {float(exact)!r}")
            for name, v in alternatives(A, fmt).items():
                if bits(v, fmt) != bits(r, fmt):
                    w(f"alt {fmt} {seed} {name} {hx(v, fmt)}")
    print("\n".join(out))


if __name__ == "__main__":
    main()
