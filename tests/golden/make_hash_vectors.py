"""Writes tests/golden/hash_vectors.txt from the ORACLE only (oracle/dyc_oracle.c).

Each row: key x_0..x_5 t1 t2 for d = 4 (s = 0 first layer, s = 1..4 subtables,
s = 5 shard), with hash constants drawn from SplitMix64(seed) (DESIGN.md §2,
reading Q1/Q2 of SURVEY.md §8(c)).  The CUDA library is checked against this
file in tests/test_gpu_parity.py; it never writes it.

    python tests/golden/make_hash_vectors.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402

SEED = 0x5EED0001
KEYS = [0, 1, 2, 3, 7, 255, 256, 65535, 65536, 0x7FFFFFFF, 0x80000000, 0xFFFFFFFA,
        0xFFFFFFFB, 0xFFFFFFFC, 0xFFFFFFFE, 0x12345678, 0xDEADBEEF, 0xCAFEBABE]


def main():
    o = oracle.OracleTable(d=4, init_capacity=4 * 4 * 1000, seed=SEED)
    import numpy as np
    rng = np.random.Generator(np.random.PCG64(7))
    keys = KEYS + [int(x) for x in rng.integers(0, 0xFFFFFFFF, size=46, dtype=np.uint64)]
    out = os.path.join(os.path.dirname(os.path.abspath(__file__)), "hash_vectors.txt")
    with open(out, "w") as f:
        f.write("# DyCuckoo hash test vectors (d = 4), written by make_hash_vectors.py from oracle/ only\n")
        f.write(f"# seed {SEED:#x}\n")
        f.write("# key x0 x1 x2 x3 x4 x5 t1 t2\n")
        for k in keys:
            xs = [o.hash_x(s, k) for s in range(6)]
            t1, t2 = o.pair(k)
            f.write(" ".join(str(v) for v in [k] + xs + [t1, t2]) + "\n")
    print("wrote", out)


if __name__ == "__main__":
    main()
