#!/usr/bin/env python
"""Run bench.py over engine/layout variants and print one line each (env SNN_CPT, --cluster-size)."""
import itertools
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(env_extra, args):
    env = dict(os.environ, **env_extra)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--cpu-images", "0", "--no-infer", "--steps", "8", *args],
                       capture_output=True, text=True, env=env)
    line = [l for l in r.stdout.splitlines() if l.startswith("{")]
    if not line:
        return None, r.stderr[-300:]
    return json.loads(line[-1]), None


if __name__ == "__main__":
    cpts = sys.argv[1].split(",") if len(sys.argv) > 1 else ["2", "4"]
    css = sys.argv[2].split(",") if len(sys.argv) > 2 else ["8", "12", "16"]
    for c, cs in itertools.product(cpts, css):
        d, err = run({"SNN_CPT": c}, ["--cluster-size", cs])
        if d is None:
            print(f"cpt={c} cs={cs}: FAILED {err}")
        else:
            print(f"cpt={c} cs={d['config']['cluster_size']} threads={d['config']['threads_per_cta']}: "
                  f"{d['value']:.1f} images/s  epochs/img {d['secondary']['epochs_per_image']:.1f}")
