"""ctypes binding of synth/libsynth.so (the GPU twin of synth/gen.py)."""
import ctypes
import os

_LIB = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libsynth.so")
_lib = None


def _get():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB):
            raise ImportError("synth/libsynth.so not built (run __graft_entry__.build())")
        lib = ctypes.CDLL(_LIB)
        lib.synth_fill.restype = ctypes.c_int
        lib.synth_fill.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64,
                                   ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        lib.synth_check.restype = ctypes.c_longlong
        lib.synth_check.argtypes = lib.synth_fill.argtypes
        _lib = lib
    return _lib


def _stream(s):
    import torch
    if s is None:
        s = torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def fill(t, seed, tensor_id, start=0, nbytes=None, stream=None):
    """Write generator bytes [start, start+nbytes) of tensor `tensor_id` into t (uint8 CUDA)."""
    n = t.numel() * t.element_size() if nbytes is None else nbytes
    rc = _get().synth_fill(t.data_ptr(), n, seed, tensor_id, start, _stream(stream))
    if rc != 0:
        raise RuntimeError("synth_fill failed: cuda error %d" % rc)


def check(t, seed, tensor_id, start=0, nbytes=None, stream=None):
    """Number of bytes of t that differ from the generator (synchronous)."""
    n = t.numel() * t.element_size() if nbytes is None else nbytes
    r = _get().synth_check(t.data_ptr(), n, seed, tensor_id, start, _stream(stream))
    if r < 0:
        raise RuntimeError("synth_check failed")
    return r


def fill_ptr(ptr, nbytes, seed, tensor_id, start=0, stream=None):
    """Write generator bytes [start, start+nbytes) of tensor `tensor_id` at
    device address `ptr` (e.g. a stash partition, for guard patterns)."""
    rc = _get().synth_fill(ptr, nbytes, seed, tensor_id, start, _stream(stream))
    if rc != 0:
        raise RuntimeError("synth_fill failed: cuda error %d" % rc)


def check_ptr(ptr, nbytes, seed, tensor_id, start=0, stream=None):
    """Number of bytes at device address `ptr` (nbytes of them) that differ
    from generator bytes [start, start+nbytes) of tensor `tensor_id`."""
    r = _get().synth_check(ptr, nbytes, seed, tensor_id, start, _stream(stream))
    if r < 0:
        raise RuntimeError("synth_check failed")
    return r


def stamp(base_u64, stream=None):
    """Write %globaltimer into base_u64 (a 1-element int64 CUDA tensor)."""
    lib = _get()
    lib.synth_stamp.restype = ctypes.c_int
    lib.synth_stamp.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
    if lib.synth_stamp(base_u64.data_ptr(), _stream(stream)) != 0:
        raise RuntimeError("synth_stamp failed")


def gate(base_u64, offset_ns, stream=None):
    """Hold the stream until %globaltimer >= base + offset_ns."""
    lib = _get()
    lib.synth_gate.restype = ctypes.c_int
    lib.synth_gate.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p]
    if lib.synth_gate(base_u64.data_ptr(), int(offset_ns), _stream(stream)) != 0:
        raise RuntimeError("synth_gate failed")
