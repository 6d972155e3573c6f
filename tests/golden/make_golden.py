"""Write tests/golden/*.json — every stored value computed by oracle/ only (never the CUDA path).

PAPER.md prints no numeric results and no worked example (its figures are images), so
these fixtures are oracle regression anchors: SHA-256 digests of the bit patterns of oracle runs on
the BASELINE.json workloads' small configs, plus a few sampled cell values for readability.
Run:  python tests/golden/make_golden.py          (small cases, seconds; re-derived by the CPU suite)
      python tests/golden/make_golden.py --latency (C5a 128^3, C5b 1024^2 at 1000 iterations: ~1 min)
      python tests/golden/make_golden.py --full   (C2 16384^2 and C3 512^3 at 1000 iterations, the
                                                   full BASELINE.json workloads: ~0.3-1 h of CPU;
                                                   too slow for the CPU suite, which re-derives the
                                                   small cases only)
"""
import hashlib
import json
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, os.path.dirname(os.path.dirname(HERE)))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
from jacobi_inputs import SEED_BENCH, u12  # noqa: E402

CASES = {
    # name: (shape (z, y, x) or (y, x), iterations) — C1 of BASELINE.json and small 3D/2D anchors
    "c1_2d_256x256_u12_5c24_1000it": ((256, 256), 1000),
    "3d_34x30x40_u12_5c24_200it": ((34, 30, 40), 200),
    "2d_66x1030_u12_5c24_77it": ((66, 1030), 77),
}


# Full-size workloads (BASELINE.json configs[1], configs[2]) at their 1000 iterations: the GPU
# suite compares the CUDA path's whole field against these digests (full-length parity).
FULL = {
    "c2_2d_16384x16384_u12_5c24_1000it": ((16384, 16384), 1000),
    "c3_3d_512x512x512_u12_5c24_1000it": ((512, 512, 512), 1000),
}


# The C5 latency workloads (BASELINE.json configs[4]) at the bench's 1000 iterations, so their
# bench lines carry whole-field parity too (seconds to a minute of CPU: python make_golden.py --latency).
LATENCY = {
    "c5a_3d_128x128x128_u12_5c24_1000it": ((128, 128, 128), 1000),
    "c5b_2d_1024x1024_u12_5c24_1000it": ((1024, 1024), 1000),
}


def digest(a: np.ndarray) -> str:
    return hashlib.sha256(np.ascontiguousarray(a, dtype=np.float64).tobytes()).hexdigest()


def compute(shape, iters):
    return oracle.jacobi(u12(shape, SEED_BENCH), iters, os.cpu_count() or 1)


def main():
    full = "--full" in sys.argv
    lat = "--latency" in sys.argv
    out = {}
    for name, (shape, iters) in (FULL if full else LATENCY if lat else CASES).items():
        r = compute(shape, iters)
        mid = tuple(s // 2 for s in shape)
        out[name] = {"shape": list(shape), "iters": iters, "seed": SEED_BENCH, "sha256": digest(r),
                     "center_value": float(r[mid]), "mean": float(r.mean()),
                     "generator": "tests/golden/make_golden.py (oracle.jacobi, C oracle)"}
        print(name, out[name]["sha256"], flush=True)
    fn = "oracle_digests_full.json" if full else "oracle_digests_latency.json" if lat else "oracle_digests.json"
    with open(os.path.join(HERE, fn), "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
