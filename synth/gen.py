"""Counter-based byte generator ("Fill pattern and parity").

Word ``w`` (8 bytes, little-endian) of tensor ``t`` under seed ``s`` is

    splitmix64(s ^ (t << 40) ^ w)

with the standard splitmix64 finaliser (Steele, Lea, Flood 2014):

    z  = x + 0x9E3779B97F4A7C15
    z  = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9
    z  = (z ^ (z >> 27)) * 0x94D049BB133111EB
    z ^= z >> 31

All arithmetic is mod 2**64.  Uniform random bits are the adversarial input
for a byte copy: every fp16/fp32 NaN payload, Inf and denormal pattern shows
up, so any float conversion on the path would corrupt them (R18).
"""
import numpy as np

_C0 = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def tensor_seed(seed: int, tensor_id: int) -> int:
    """Per-tensor key ``seed ^ (tensor_id << 40)`` (mod 2**64)."""
    return (int(seed) ^ (int(tensor_id) << 40)) & 0xFFFFFFFFFFFFFFFF


def splitmix64_words(seed: int, tensor_id: int, w0: int, nwords: int) -> np.ndarray:
    """Words ``w0 .. w0+nwords-1`` of tensor ``tensor_id`` as uint64."""
    key = np.uint64(tensor_seed(seed, tensor_id))
    x = np.arange(w0, w0 + nwords, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x ^= key
        z = x + _C0
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        z ^= z >> np.uint64(31)
    return z


def splitmix64_bytes(seed: int, tensor_id: int, start: int, length: int) -> np.ndarray:
    """Bytes ``[start, start+length)`` of tensor ``tensor_id`` as a uint8 array."""
    if length <= 0:
        return np.zeros(0, dtype=np.uint8)
    w0 = start // 8
    w1 = (start + length + 7) // 8
    words = splitmix64_words(seed, tensor_id, w0, w1 - w0)
    b = words.astype("<u8").view(np.uint8)
    off = start - w0 * 8
    return b[off:off + length]
