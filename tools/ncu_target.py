#!/usr/bin/env python
"""Small profiling target: C4 network, 2 warm-up images, then ONE present_batch launch of
--images images (profile it with ncu -k regex:present_event -c 1 ...; never time under ncu)."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synthdata  # noqa: E402
import paper_conf_date_shelm19_b200 as P  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--images", type=int, default=32)
ap.add_argument("--n-exc", type=int, default=6400)
a = ap.parse_args()
net = P.Network(784, a.n_exc, 2, P.preset("2b", membrane_mode=0))
imgs = synthdata.images(a.images + 2, "fashion")
seeds = synthdata.seeds(a.images + 2, 1)
net.present_batch(imgs[:2], 350, seeds[:2])
net.present_batch(imgs[2:], 350, seeds[2:])
print("ok", net.stats()[:2])
