"""Plain numpy statement of the configuration hash of include/aceso.h (aceso_hash) and of the
visited-set semantics (aceso_dedup): test reference, shares nothing with csrc/."""
import numpy as np

SEED, POS = 0x243F6A8885A308D3, 0x9E3779B97F4A7C15


def _mix(x):
    x = x ^ (x >> np.uint64(30))
    x = x * np.uint64(0xBF58476D1CE4E5B9)
    x = x ^ (x >> np.uint64(27))
    x = x * np.uint64(0x94D049BB133111EB)
    return x ^ (x >> np.uint64(31))


def config_hash(codes: np.ndarray, hdr: np.ndarray) -> np.ndarray:
    """codes [n][L] u8 row-major, hdr [n] u64 -> [n] u64 (include/aceso.h, aceso_hash)."""
    n, L = codes.shape
    m = (L + 8 + 7) // 8
    buf = np.zeros((n, 8 * m), np.uint8)
    buf[:, :L] = codes
    buf[:, L:L + 8] = np.ascontiguousarray(hdr, np.uint64).view(np.uint8).reshape(n, 8)
    words = buf.view("<u8")
    with np.errstate(over="ignore"):
        s = np.zeros(n, np.uint64)
        for i in range(m):
            s = s + _mix(words[:, i] ^ (np.uint64(i + 1) * np.uint64(POS)))
        h = _mix(np.uint64(SEED) + s)
    h[h == 0] = 1
    return h


class VisitedReference:
    """First occurrence across calls: a hash is new iff never seen in an earlier call and
    not at a lower index of this call."""

    def __init__(self):
        self.seen = set()

    def insert(self, hashes: np.ndarray) -> np.ndarray:
        dup = np.zeros(len(hashes), np.uint8)
        this = set()
        for i, h in enumerate(hashes.tolist()):
            if h in self.seen or h in this:
                dup[i] = 1
            this.add(h)
        self.seen |= this
        return dup
