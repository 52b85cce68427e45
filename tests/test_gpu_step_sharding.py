"""Column-sharded per-step engine (NEXT-2 at C4 scale) against the unsharded
oracle (needs a B200).  On the per-step engine every step's WTA summary of each shard's cluster (best key for
HARD, spiker count for LAYER) goes to every shard's device-memory mailbox and every shard applies the same
reduction.  This is what lets a 784 -> 6400 network with 16-bit codes (10 MB, R27) or binary32 conductances
(20 MB, R28) learn: 4 / 7 clusters of <= 16 CTAs on one B200, presented in ONE snn_present_many launch.
The union of the shards must equal the oracle: codes / conductances, rasters, per-image spike counts, state
and counters (membranes within 1e-5 relative in fp32 mode)."""
import numpy as np
import pytest

import synthdata
from oracle import oracle as O

from test_gpu_sharding import _compare

pytestmark = pytest.mark.gpu


def _step_shards(n_in, n_exc, bits, p, world):
    import paper_conf_date_shelm19_b200 as P
    sh = [P.Network(n_in, n_exc, bits, P.params_from_dict(p, engine=1), shard=(r, world)) for r in range(world)]
    assert all(s.info()["engine"] == 1 for s in sh)
    P.link_shards(sh)
    return sh


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("wta,stdp", [(0, 0), (1, 0), (0, 1)])
def test_step_sharded_784x400_8bit(gpu, world, wta, stdp):
    p = O.params("8b", wta_mode=wta, stdp_mode=stdp, membrane_mode=1, init_seed=3)
    sh = _step_shards(784, 400, 8, p, world)
    o = O.OracleNet(784, 400, 8, p)
    _compare(sh, o, synthdata.images(2, "mnist", start=300), 150, synthdata.seeds(2, base_seed=41), 784, 400, 1)
    assert int(o.stats()[1]) > 0


def test_step_sharded_16bit_784x800(gpu):
    p = O.params("16b", rounding=2, membrane_mode=0, init_seed=4)
    sh = _step_shards(784, 800, 16, p, 2)
    o = O.OracleNet(784, 800, 16, p)
    _compare(sh, o, synthdata.images(2, "fashion", start=10), 120, synthdata.seeds(2, base_seed=42), 784, 800, 0)


def test_step_sharded_16bit_C4_784x6400(gpu):
    """NEXT-2 at the C4 network: 784 -> 6400 with 16-bit codes (10 MB) as 4 shards x 16 CTAs."""
    import paper_conf_date_shelm19_b200 as P
    p = O.params("16b", rounding=2, membrane_mode=1, init_seed=5)
    with pytest.raises(P.SnnError):                  # one cluster cannot hold it
        P.Network(784, 6400, 16, P.params_from_dict(p))
    sh = _step_shards(784, 6400, 16, p, 4)
    o = O.OracleNet(784, 6400, 16, p)
    _compare(sh, o, synthdata.images(1, "fashion", start=20), 60, synthdata.seeds(1, base_seed=43), 784, 6400, 1)
    assert int(o.stats()[1]) > 0


def test_step_sharded_fp32_C4_784x6400(gpu):
    """NEXT-2 at the C4 network with binary32 conductances (20 MB, R28) as 7 shards of 15-16 CTAs (7 clusters of
    16 CTAs is what a B200's GPCs hold at once)."""
    p = O.params("16b", init_seed=6)
    sh = _step_shards(784, 6400, 32, p, 7)
    o = O.OracleNet(784, 6400, 32, p)
    _compare(sh, o, synthdata.images(1, "fashion", start=21), 60, synthdata.seeds(1, base_seed=44), 784, 6400, 0)
    assert int(o.stats()[1]) > 0


def test_step_sharded_fp32_deterministic_layer(gpu):
    p = O.params("16b", stdp_mode=1, wta_mode=1, init_seed=7)
    sh = _step_shards(784, 640, 32, p, 3)
    o = O.OracleNet(784, 640, 32, p)
    _compare(sh, o, synthdata.images(2, "mnist", start=30), 120, synthdata.seeds(2, base_seed=45), 784, 640, 0)
