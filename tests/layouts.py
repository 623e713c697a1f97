"""The layout families of PAPER.md L27 (Section I), as test data.

"For contractions of two 3D tensors, and a single contraction (summation) index, there
are 846 (3! x 3! x 4!) possible cases.  If the contraction has two contraction indices,
there are 72 cases."  The product 3!*3!*4! is 864 (reading R10: "846" is a
typo); with two contraction indices C is 2D and the count is 3!*3!*2! = 72.
"""
from itertools import permutations


def layouts_one_contraction():
    """C 4D = A 3D x B 3D with one contraction index k: 3! * 3! * 4! = 864 strings."""
    out = []
    for a in permutations("abk"):
        for b in permutations("cdk"):
            for c in permutations("abcd"):
                out.append("".join(c) + "-" + "".join(a) + "-" + "".join(b))
    return out


def layouts_two_contractions():
    """C 2D = A 3D x B 3D with two contraction indices k, l: 3! * 3! * 2! = 72."""
    out = []
    for a in permutations("akl"):
        for b in permutations("bkl"):
            for c in permutations("ab"):
                out.append("".join(c) + "-" + "".join(a) + "-" + "".join(b))
    return out


# pairwise DISTINCT small primes, so a transposed index cannot alias another one (no two
# indices of any layout share an extent: a swapped pair of indices changes the shape)
PRIME_EXT = {"a": 2, "b": 3, "c": 5, "d": 7, "k": 11, "l": 13}
assert len(set(PRIME_EXT.values())) == len(PRIME_EXT)
