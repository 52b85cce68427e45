"""Column-sharded event engine against the unsharded oracle (needs a
B200).  A network's columns are split over `world` shard handles (include/snn.h
snn_create_shard); per epoch the shards exchange their 16-byte summaries through device-memory
mailboxes.  On one GPU the shards are linked in-process and presented in ONE launch
(snn_present_many keeps every shard co-resident); the IPC test runs two processes on the same
GPU, each owning one shard, connected with CUDA IPC handles exactly as bench.py's multi-rank
shard mode does across GPUs.  The union of the shards must equal the oracle bit for bit:
conductance codes, output rasters, per-image spike counts, state and counters."""
import os

import numpy as np
import pytest

import synthdata
from oracle import oracle as O

pytestmark = pytest.mark.gpu


def _shards(n_in, n_exc, bits, p, world):
    import paper_conf_date_shelm19_b200 as P
    sh = [P.Network(n_in, n_exc, bits, P.params_from_dict(p), shard=(r, world)) for r in range(world)]
    P.link_shards(sh)
    return sh


def _cat_raster(shards, T):
    return np.concatenate([O.unpack_bits(s.spikes(), s.n_exc)[:T] for s in shards], axis=1)


def _compare(shards, o, images, T, seeds, n_in, n_exc, mode):
    import paper_conf_date_shelm19_b200 as P
    world = len(shards)
    for img, sd in zip(images, seeds):
        for s in shards:
            s.reset_stats()
        P.present_many(shards, [img[None]] * world, T, [np.array([sd], np.uint64)] * world)
        o.present(img, T, int(sd))
        assert np.array_equal(_cat_raster(shards, T), O.unpack_bits(o.spikes(), n_exc)), "output raster"
        assert np.array_equal(np.concatenate([s.weights() for s in shards], axis=1), o.weights()), "codes"
        so = o.stats()
        st = [s.stats() for s in shards]
        for k in (0, 1):                                   # network-wide counters: identical on every shard
            assert all(int(x[k]) == int(so[k]) for x in st), k
        for k in (2, 3, 4, 5):                             # per-shard trials / events add up
            assert sum(int(x[k]) for x in st) == int(so[k]), k
        ref = O.unpack_state(o.state(), n_in, n_exc)
        parts = [O.unpack_state(s.state(), n_in, s.n_exc) for s in shards]
        for k in ("cnt", "last_post"):
            assert np.array_equal(np.concatenate([x[k] for x in parts]), ref[k]), k
        for x in parts:
            assert np.array_equal(x["last_pre"], ref["last_pre"])
        v = np.concatenate([x["v"] for x in parts])
        if mode == 1:
            assert np.array_equal(v, ref["v"])
        else:
            np.testing.assert_allclose(v, ref["v"], rtol=1e-5, atol=0)


def test_shard_column_ranges(gpu):
    import paper_conf_date_shelm19_b200 as P
    p = P.params_from_dict(O.params("8b"))
    G = (1000 + 31) // 32
    for world in (1, 2, 3, 5, 8):
        sh = [P.Network(784, 1000, 8, p, shard=(r, world)) for r in range(world)]
        los = [s.info()["col_base"] for s in sh]
        assert los == [32 * (r * G // world) for r in range(world)]
        assert sum(s.n_exc for s in sh) == 1000
        assert all(s.info()["n_exc_total"] == 1000 and s.info()["world"] == world for s in sh)
        shapes = {(s.info()["cluster_size"], s.info()["threads"], s.info()["smem_bytes"]) for s in sh}
        assert len(shapes) == 1, "shards of one world share one launch shape"


@pytest.mark.parametrize("world", [2, 3, 4])
@pytest.mark.parametrize("mode", [0, 1])
def test_sharded_C1_784x100_8bit(gpu, world, mode):
    p = O.params("8b", membrane_mode=mode, init_seed=1)
    sh = _shards(784, 100, 8, p, world)
    o = O.OracleNet(784, 100, 8, p)
    assert np.array_equal(np.concatenate([s.weights() for s in sh], axis=1), o.weights()), "init (R4, global j)"
    _compare(sh, o, synthdata.images(6, "mnist"), 100, synthdata.seeds(6, base_seed=1), 784, 100, mode)
    assert o.stats()[1] > 0


@pytest.mark.parametrize("stdp,rounding", [(0, 1), (1, 2)])
def test_sharded_C2_784x400_layer(gpu, stdp, rounding):
    p = O.params("8b", wta_mode=1, stdp_mode=stdp, rounding=rounding, membrane_mode=1, init_seed=2)
    sh = _shards(784, 400, 8, p, 3)
    o = O.OracleNet(784, 400, 8, p)
    _compare(sh, o, synthdata.images(2, "mnist", start=100), 350, synthdata.seeds(2, base_seed=2), 784, 400, 1)
    assert o.stats()[1] > 0


@pytest.mark.parametrize("mode,wta", [(0, 0), (1, 1)])
def test_sharded_inh_hold(gpu, mode, wta):
    p = O.params("8b", inh_mode=1, wta_mode=wta, membrane_mode=mode, init_seed=12)
    sh = _shards(784, 400, 8, p, 2)
    o = O.OracleNet(784, 400, 8, p)
    _compare(sh, o, synthdata.images(2, "mnist", start=40), 250, synthdata.seeds(2, 12), 784, 400, mode)


def test_sharded_undo_log_overflow(gpu):
    """Log-full stops on one shard must stop the others through the cross-shard flag / summary."""
    p = O.params("2b", f_min_hz=200.0, f_max_hz=1000.0, gamma_dep=1.0, tau_dep=50.0, v_spike=0.5,
                 membrane_mode=1, init_seed=13)
    sh = _shards(784, 256, 2, p, 2)
    o = O.OracleNet(784, 256, 2, p)
    _compare(sh, o, synthdata.images(2, "fashion", start=3), 120, synthdata.seeds(2, 13), 784, 256, 1)
    assert sum(int(s.stats()[9]) for s in sh) > 0, "undo-log overflow path not exercised"


@pytest.mark.parametrize("world", [2, 4])
def test_sharded_C4_784x6400_2bit(gpu, world):
    """The bench workload split over `world` shards, against the ORACLE: one image presented alone, then
    a batch of 4 images in one launch (the oracle presents them one by one)."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("2b", membrane_mode=0, init_seed=1)
    sh = _shards(784, 6400, 2, p, world)
    o = O.OracleNet(784, 6400, 2, p)
    imgs = synthdata.images(5, "fashion")
    seeds = synthdata.seeds(5, base_seed=1)
    _compare(sh, o, imgs[:1], 350, seeds[:1], 784, 6400, 0)
    for s in sh:
        s.reset_stats()
    P.present_many(sh, [imgs[1:]] * world, 350, [seeds[1:]] * world)
    post = 0
    for img, sd in zip(imgs[1:], seeds[1:]):
        o.present(img, 350, int(sd))
        post += int(o.stats()[1])
    assert np.array_equal(np.concatenate([s.weights() for s in sh], axis=1), o.weights())
    assert np.array_equal(_cat_raster(sh, 350), O.unpack_bits(o.spikes(), 6400))
    assert all(int(s.stats()[1]) == post for s in sh)
    ref = O.unpack_state(o.state(), 784, 6400)
    parts = [O.unpack_state(s.state(), 784, s.n_exc) for s in sh]
    for k in ("cnt", "last_post"):
        assert np.array_equal(np.concatenate([x[k] for x in parts]), ref[k]), k
    np.testing.assert_allclose(np.concatenate([x["v"] for x in parts]), ref["v"], rtol=1e-5, atol=0)


def test_shard_api_errors(gpu):
    import paper_conf_date_shelm19_b200 as P
    p = O.params("8b", membrane_mode=1)
    pp = P.params_from_dict(p)
    with pytest.raises(P.SnnError) as e:                  # 4 column groups cannot feed 5 shards
        P.Network(784, 100, 8, pp, shard=(0, 5))
    assert e.value.rc == -1
    with pytest.raises(P.SnnError):                       # bits > 8 shard on the per-step engine only
        P.Network(784, 100, 16, P.params_from_dict(O.params("16b"), engine=2), shard=(0, 2))
    a, b = (P.Network(784, 100, 8, pp, shard=(r, 2)) for r in range(2))
    img = synthdata.images(1, "mnist")[0]
    with pytest.raises(P.SnnError):                       # not connected yet
        a.present(img, 10, 1)
    P.link_shards([a, b])
    with pytest.raises(P.SnnError):                       # same-device shards run in one launch only
        a.present(img, 10, 1)
    with pytest.raises(P.SnnError):                       # its world must be complete
        P.present_many([a], [img[None]], 10, [np.array([1], np.uint64)])
    P.present_many([a, b], [img[None]] * 2, 10, [np.array([1], np.uint64)] * 2)


# ------------------------------------------------------------------ two processes, CUDA IPC mailboxes
def _ipc_worker(rank, world, tmp, p, imgs, seeds, T, bits=8, engine=0):
    import torch
    import paper_conf_date_shelm19_b200 as P
    torch.cuda.set_device(0)
    net = P.Network(784, 128, bits, P.params_from_dict(p, engine=engine), shard=(rank, world))
    with open(os.path.join(tmp, f"h{rank}.tmp"), "wb") as f:
        f.write(net.ipc_handle())
    os.rename(os.path.join(tmp, f"h{rank}.tmp"), os.path.join(tmp, f"h{rank}.bin"))
    import time
    t_end = time.time() + 120
    while not all(os.path.exists(os.path.join(tmp, f"h{r}.bin")) for r in range(world)):
        assert time.time() < t_end, "peer never published its handle"
        time.sleep(0.05)
    handles = [open(os.path.join(tmp, f"h{r}.bin"), "rb").read() for r in range(world)]
    net.connect(handles)
    counts = np.zeros(len(imgs), np.int32)
    net.present_batch(imgs, T, seeds, counts)
    np.save(os.path.join(tmp, f"w{rank}.npy"), net.weights())
    np.save(os.path.join(tmp, f"c{rank}.npy"), counts)


def test_sharded_two_processes_ipc(gpu, tmp_path):
    """The multi-rank protocol proper: two processes, one shard each, mailboxes opened with CUDA
    IPC (on one GPU the two kernels are time-sliced; across GPUs they run side by side)."""
    import torch.multiprocessing as mp
    p = O.params("8b", membrane_mode=1, init_seed=3, f_min_hz=5.0, f_max_hz=78.0)
    imgs = synthdata.images(2, "mnist", start=5)
    seeds = synthdata.seeds(2, base_seed=3)
    T = 60
    ctx = mp.get_context("spawn")
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, str(tmp_path), p, imgs, seeds, T)) for r in range(2)]
    for x in procs:
        x.start()
    for x in procs:
        x.join(timeout=240)
    for x in procs:
        if x.is_alive():
            x.kill()
    assert all(x.exitcode == 0 for x in procs), [x.exitcode for x in procs]
    o = O.OracleNet(784, 128, 8, p)
    oc = []
    for img, sd in zip(imgs, seeds):
        o.present(img, T, int(sd))
        oc.append(int(O.unpack_bits(o.spikes(), 128).sum()))
    w = np.concatenate([np.load(tmp_path / f"w{r}.npy") for r in range(2)], axis=1)
    assert np.array_equal(w, o.weights())
    for r in range(2):
        assert np.load(tmp_path / f"c{r}.npy").tolist() == oc


def test_step_sharded_two_processes_ipc(gpu, tmp_path):
    """The per-step engine's shard exchange (one mailbox round per step) between two processes over CUDA IPC,
    16-bit codes (R27): what a 784 -> 6400 16-bit network does across GPUs, here time-sliced on one GPU."""
    import torch.multiprocessing as mp
    p = O.params("16b", membrane_mode=1, rounding=2, init_seed=4, f_min_hz=5.0, f_max_hz=78.0)
    imgs = synthdata.images(2, "mnist", start=6)
    seeds = synthdata.seeds(2, base_seed=5)
    T = 40
    ctx = mp.get_context("spawn")
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, str(tmp_path), p, imgs, seeds, T, 16, 1)) for r in range(2)]
    for x in procs:
        x.start()
    for x in procs:
        x.join(timeout=240)
    for x in procs:
        if x.is_alive():
            x.kill()
    assert all(x.exitcode == 0 for x in procs), [x.exitcode for x in procs]
    o = O.OracleNet(784, 128, 16, p)
    oc = []
    for img, sd in zip(imgs, seeds):
        o.present(img, T, int(sd))
        oc.append(int(O.unpack_bits(o.spikes(), 128).sum()))
    w = np.concatenate([np.load(tmp_path / f"w{r}.npy") for r in range(2)], axis=1)
    assert np.array_equal(w, o.weights())
    for r in range(2):
        assert np.load(tmp_path / f"c{r}.npy").tolist() == oc


@pytest.mark.parametrize("k", range(12))
def test_sharded_lean_fuzz(gpu, k):
    """Randomised column-sharded networks on the lean kernel (the paper's default mode): world 2-4, widths,
    column counts, rates and refractory/inhibition lengths; the union of the shards against the oracle."""
    rng = np.random.default_rng(500 + k)
    bits = int(rng.choice([2, 4, 8]))
    world = int(rng.choice([2, 3, 4]))
    n_exc = 32 * world * int(rng.integers(1, 5))
    fmin, fmax = [(1.0, 22.0), (5.0, 78.0)][int(rng.integers(2))]
    p = O.params({2: "2b", 4: "4b", 8: "8b"}[bits], membrane_mode=int(rng.integers(2)), init_seed=int(rng.integers(1, 99)),
                 f_min_hz=fmin, f_max_hz=fmax, t_ref_steps=int(rng.choice([2, 5, 10])), t_inh_steps=int(rng.choice([3, 10])),
                 v_spike=float(rng.choice([2.0, 4.0])))
    sh = _shards(784, n_exc, bits, p, world)
    assert all(s.info()["lean"] == 1 for s in sh)
    o = O.OracleNet(784, n_exc, bits, p)
    kind = str(rng.choice(["mnist", "fashion"]))
    _compare(sh, o, synthdata.images(2, kind, start=int(rng.integers(5000))), 150, synthdata.seeds(2, k + 3), 784, n_exc,
             p["membrane_mode"])
