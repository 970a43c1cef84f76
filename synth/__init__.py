"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no planning, no striping,
no copying): only

* ``splitmix64_bytes`` -- the counter-based byte generator every tensor of every
  workload is filled with (SURVEY.md §8(d) "Fill pattern"), and
* ``workloads`` -- the tensor-size lists of BASELINE.json's five configs.

Both sides regenerate the same bytes from (seed, tensor id, byte range), so a
GB-scale tensor can be checked window by window without holding a host copy.
The GPU-side twin of the generator lives in ``synth/fill.cu`` (built into
``synth/libsynth.so``); it shares no code with the product library either.
"""
from .gen import splitmix64_words, splitmix64_bytes, tensor_seed  # noqa: F401
from . import workloads  # noqa: F401
