"""ORACLE (test infrastructure only) -- byte model of swap-out and swap-in.

D2D swap is a lossless move (MPress "does not affect" accuracy), so the
result has a plain definition (SURVEY.md §8(c) "Plain definition", step 8):

  swap-out: for every stripe (i, p, src_off, dst_off, len)
            stash[p][dst_off : dst_off+len] = tensor[i][src_off : src_off+len]
  swap-in:  dst[i][src_off : src_off+len] = stash[p][dst_off : dst_off+len]

guided by the metadata table of P:211 (here: the plan's stripe list).  Bytes
of a peer's stash that no stripe covers (the <=255 B alignment padding, R6)
are unspecified; ``swap_out`` reports them in a ``defined`` mask so parity
tests compare only the defined bytes.
"""
import numpy as np

POISON = 0xA5


def stash_sizes(plan):
    """Bytes of the virtual batch that live on each peer (plan['peer_bytes'])."""
    return list(plan["peer_bytes"])


def swap_out(plan, tensors):
    """Return {peer: (stash uint8[peer_bytes], defined bool[peer_bytes])}."""
    assert len(tensors) == len(plan["sizes"])
    out = {}
    for p, nbytes in enumerate(plan["peer_bytes"]):
        if nbytes > 0:
            out[p] = (np.full(nbytes, POISON, dtype=np.uint8),
                      np.zeros(nbytes, dtype=bool))
    for (i, p, src_off, dst_off, ln) in plan["stripes"]:
        t = np.asarray(tensors[i], dtype=np.uint8).reshape(-1)
        assert t.size == plan["sizes"][i]
        stash, defined = out[p]
        stash[dst_off:dst_off + ln] = t[src_off:src_off + ln]
        defined[dst_off:dst_off + ln] = True
    return out


def swap_in(plan, stash):
    """Rebuild every tensor from the peers' stash (one new buffer per tensor)."""
    dst = [np.full(s, POISON ^ 0xFF, dtype=np.uint8) for s in plan["sizes"]]
    for (i, p, src_off, dst_off, ln) in plan["stripes"]:
        dst[i][src_off:src_off + ln] = stash[p][0][dst_off:dst_off + ln]
    return dst
