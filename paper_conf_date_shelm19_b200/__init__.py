"""B200-native (sm_100a) simulate-and-learn loop of She, Long & Mukhopadhyay (DATE'19).

The compute path is the CUDA library libsnn_b200.so behind the C ABI include/snn.h; this
package is the thin ctypes binding (snn.py).  See DESIGN.md.
"""
from .snn import (Network, SnnError, SnnParams, link_shards, params_from_dict, present_many, infer_many, preset, lib,  # noqa: F401
                  SNN_RASTER_INPUT, SNN_KEEP_STATE, SNN_RECORD_INPUT, SNN_ASYNC, EXPORTS)

__all__ = ["Network", "SnnError", "SnnParams", "params_from_dict", "present_many", "infer_many", "preset", "lib"]
