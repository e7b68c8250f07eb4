"""Writes tests/golden/gen_checksums.json from the ORACLE ONLY (oracle/ -- O-GEN, docs/GENERATOR.md).

Run: python -m tests.golden.make_golden     (re-run only when the generator spec changes; say why in the commit)
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import workloads as W  # noqa: E402

OUT = os.path.join(os.path.dirname(os.path.abspath(__file__)), "gen_checksums.json")


def _fnv1a64(b: bytes) -> int:
    h = 0xCBF29CE484222325
    a = np.frombuffer(b, dtype=np.uint8)
    # vectorised FNV-1a is sequential; chunk through python ints in blocks for moderate sizes
    for byte in a.tolist():
        h ^= byte
        h = (h * 0x100000001B3) & 0xFFFFFFFFFFFFFFFF
    return h


def system_checksums(S):
    out = {}
    for name in ("vals", "mA", "mT", "iC", "b", "c_ptr", "c_col", "c_val"):
        arr = np.ascontiguousarray(getattr(S, name))
        out[name] = format(_fnv1a64(arr.tobytes()), "016x")
    out["row_ptr"] = format(_fnv1a64(S.row_ptr.tobytes()), "016x")
    return out


def golden_cases():
    return {
        "micro": W.micro(),
        "micro_noglob": W.micro(n_glob=0, seed=5),
        "micro_constr": W.micro(n_stars=9, obs=20, n_ext=4, seed=9),
        "micro_planted": W.micro(seed=13, b_mode=1, noise=0.25),
        "C1_head": W.C1.replace(n_stars=40, n_obs=800),
    }



def main():
    gold = {name: system_checksums(oracle.System(w)) for name, w in golden_cases().items()}
    with open(OUT, "w") as f:
        json.dump(gold, f, indent=1, sort_keys=True)
    print("wrote", OUT)


if __name__ == "__main__":
    main()
