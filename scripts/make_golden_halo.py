"""Write tests/golden/halo_eq8_eq9.txt from the paper's summation definitions
(Eq 8: f(k) = sum_{i=0}^{k-1} 2^i; Eq 9, P:421-427:
g(k) = k f(k) - sum_{i=0}^{k} f(i)) and Table I (cache 3 f(k) <= 3*2^k).
Pure Python; calls nothing from the CUDA path or the oracle."""
import os

out = os.path.join(os.path.dirname(__file__), "..", "tests", "golden", "halo_eq8_eq9.txt")


def f(k):
    return sum(2 ** i for i in range(k))


def g(k):
    return k * f(k) - sum(f(i) for i in range(k + 1))


with open(out, "w") as fh:
    fh.write("# Eq 8 f(k) and Eq 9 g(k) by their summation definitions (PAPER.md P:413-427);\n")
    fh.write("# Table I cache 3*f(k) (P:627-631). Fig 7 (P:411): k=1 -> 1 halo row; k=2 -> 3 halo rows\n")
    fh.write("# and 2 redundant eliminations (e'2, e'3).  Columns: k f g cache3f\n")
    for k in range(0, 21):
        fh.write(f"{k} {f(k)} {g(k)} {3 * f(k)}\n")
