"""Independent numpy re-implementation of the library's internal priority bijection
(reading 16: 4-round keyed Feistel on 2*half >= log2(n) bits, cycle walking).
Used only to map the GPU's per-iteration signatures (which are priorities) back onto the
oracle's run on the relabelled graph; it holds none of the SCC method's arithmetic."""
import numpy as np

KEYS = (0x3C6EF372, 0xA54FF53A, 0x510E527F, 0x9B05688C)


def _hash(x):
    x = (x * np.uint32(0x9E3779B1)).astype(np.uint32)
    x ^= x >> np.uint32(15)
    x = (x * np.uint32(0x85EBCA77)).astype(np.uint32)
    x ^= x >> np.uint32(13)
    return x


def prio(n: int, v=None) -> np.ndarray:
    """pi(v) for v in [0, n) (or the given vector)."""
    bits = 1
    while bits < 32 and (1 << bits) < n:
        bits += 1
    half = (bits + 1) // 2
    mask = np.uint32((1 << half) - 1)
    x = np.arange(n, dtype=np.uint32) if v is None else np.asarray(v, dtype=np.uint32).copy()
    out = x.copy()
    todo = np.ones(x.shape, dtype=bool)
    with np.errstate(over="ignore"):
        while todo.any():
            y = out[todo]
            L, R = y >> np.uint32(half), y & mask
            for k in KEYS:
                L, R = R, L ^ (_hash(R ^ np.uint32(k)) & mask)
            y = (L << np.uint32(half)) | R
            out[todo] = y
            todo[todo] = y >= n
    return out.astype(np.int64)
