#!/usr/bin/env python
"""Profiling target for the per-step engine: 784 -> 400 with 16-bit codes (NEXT-2, R27) or binary32 conductances
(R28), 2 warm-up images then ONE present_batch launch of --images images (profile with
ncu -k regex:present_kernel --launch-skip 1 -c 1; never time under ncu)."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402
import paper_conf_date_shelm19_b200 as P  # noqa: E402
from oracle import oracle as O  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--images", type=int, default=4)
ap.add_argument("--bits", type=int, default=16)
a = ap.parse_args()
net = P.Network(784, 400, a.bits, P.params_from_dict(O.params("16b", rounding=2 if a.bits == 16 else 1)))
imgs = synthdata.images(a.images + 2, "mnist")
seeds = synthdata.seeds(a.images + 2, 1)
net.present_batch(imgs[:2], 350, seeds[:2])
net.present_batch(imgs[2:], 350, seeds[2:])
print("ok", net.info()["cluster_size"], net.stats()[:2])
