"""The C ABI from plain C (examples/present_c.c): no Python binding, no PyTorch in the process.

The header must compile as C99 with warnings as errors and the program must link against the in-tree
library (CPU, no GPU needed); on a B200 the program's outputs (codes, per-image spike counts, last raster,
counters) must equal the oracle's for the same images and seeds."""
import os
import subprocess

import numpy as np
import pytest

import synthdata
from oracle import oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIBDIR = os.path.join(ROOT, "paper_conf_date_shelm19_b200")


def _build(tmp_path):
    exe = str(tmp_path / "present_c")
    subprocess.run(["gcc", "-std=c99", "-Wall", "-Wextra", "-Werror", "-I", os.path.join(ROOT, "include"),
                    os.path.join(ROOT, "examples", "present_c.c"), "-L", LIBDIR, "-lsnn_b200",
                    f"-Wl,-rpath,{LIBDIR}", "-o", exe], check=True)
    return exe


def test_c_program_builds_and_links(tmp_path):
    exe = _build(tmp_path)
    r = subprocess.run([exe], capture_output=True, text=True)
    assert r.returncode == 2 and "usage" in r.stderr


@pytest.mark.gpu
@pytest.mark.parametrize("n_exc,bits,preset,T,n,kind", [(100, 8, 2, 100, 3, "mnist"), (6400, 2, 0, 350, 2, "fashion")])
def test_c_program_matches_oracle(gpu, tmp_path, n_exc, bits, preset, T, n, kind):
    exe = _build(tmp_path)
    imgs = synthdata.images(n, kind, start=40)
    seeds = synthdata.seeds(n, base_seed=17)
    imgs.tofile(tmp_path / "imgs.u8")
    seeds.astype(np.uint64).tofile(tmp_path / "seeds.u64")
    out = str(tmp_path / "out")
    r = subprocess.run([exe, "784", str(n_exc), str(bits), str(preset), str(T), str(n), str(tmp_path / "imgs.u8"),
                        str(tmp_path / "seeds.u64"), out], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    o = O.OracleNet(784, n_exc, bits, O.params({0: "2b", 2: "8b"}[preset]))
    want = []
    for x, s in zip(imgs, seeds):
        o.present(x, T, int(s))
        want.append(int(O.unpack_bits(o.spikes(), n_exc).sum()))
    assert np.fromfile(out + ".counts", np.int32).tolist() == want
    assert np.array_equal(np.fromfile(out + ".codes", np.uint8).reshape(784, n_exc), o.weights())
    assert np.array_equal(np.fromfile(out + ".raster", np.uint32).reshape(T, -1), o.spikes())
    st = np.fromfile(out + ".stats", np.uint64)
    assert int(st[1]) == sum(want)
