"""Writes tests/golden/hash_vectors_wide.txt from the ORACLE only
(oracle/dyw_oracle.c): the 64-bit-key hash of reading Q33,
x_s(k) = (c_s*hi(k) + a_s*lo(k) + b_s) mod p, for d = 4 (s = 0 first layer,
s = 1..4 subtables, s = 5 shard), constants from SplitMix64(seed).  The CUDA
library is checked against this file (tests/test_gpu_wide.py); it never writes it.

    python tests/golden/make_hash_vectors_wide.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402

SEED = 0x5EED0001
KEYS = [0, 1, 0xFFFFFFFF, 0x100000000, 0x100000001, 0xFFFFFFFB00000000, 0xFFFFFFFA, 0xFFFFFFFB,
        0x123456789ABCDEF0, 0xDEADBEEFCAFEBABE, 0x8000000000000000, 0x7FFFFFFFFFFFFFFF,
        0xFFFFFFFFFFFFFFFE, 0xFFFFFFFEFFFFFFFF]


def main():
    o = oracle.OracleWideTable(d=4, init_capacity=4 * 16 * 1000, seed=SEED, bucket_slots=16, value_words=1)
    rng = np.random.Generator(np.random.PCG64(11))
    keys = KEYS + [int(x) for x in rng.integers(0, 0xFFFFFFFFFFFFFFFF, size=50, dtype=np.uint64)]
    out = os.path.join(os.path.dirname(os.path.abspath(__file__)), "hash_vectors_wide.txt")
    with open(out, "w") as f:
        f.write("# DyCuckoo wide-key hash test vectors (d = 4, reading Q33), "
                "written by make_hash_vectors_wide.py from oracle/ only\n")
        f.write(f"# seed {SEED:#x}\n")
        f.write("# key x0 x1 x2 x3 x4 x5 t1 t2\n")
        for k in keys:
            xs = [o.hash_x(s, k) for s in range(6)]
            t1, t2 = o.pair(k)
            f.write(" ".join(str(v) for v in [k] + xs + [t1, t2]) + "\n")
    print("wrote", out)


if __name__ == "__main__":
    main()
