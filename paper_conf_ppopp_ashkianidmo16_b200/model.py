"""Byte model of the multisplit hot path (host logic, no device code).

Speed of light, §6.2.2: one read of every key before
the global operation, then one read of every key (key-value: pair) and one
write of it after -- 3 accesses per key (12 B) key-only, 5 (20 B) key-value.
Precomputed ids (MS_IDS, id_bytes per id): the pass before the global
operation needs only the ids (id_bytes instead of the 4-byte key), the pass
after reads the id next to the key: 2*id_bytes + 8 B (key-only) / + 16 B.
The 3-kernel form adds the H / G round trips (write H in K1, read+write it in
K2, read G in K3): 16*m/T bytes per key (DESIGN.md §"Kernels").
"""


def algorithmic_bytes_per_key(with_values: bool, id_bytes: int = 0) -> int:
    """Paper's speed-of-light bytes per key: 12 (key-only) / 20 (key-value); with precomputed ids
    (id_bytes > 0) 8 / 16 + 2*id_bytes."""
    pre, post = pass_bytes_per_key(with_values, id_bytes)
    return pre + post


def pass_bytes_per_key(with_values: bool, id_bytes: int = 0):
    """Algorithmic bytes per key of each pass: (pre-scan, post-scan)."""
    pre = id_bytes if id_bytes else 4
    post = (16 if with_values else 8) + id_bytes
    return pre, post


def hg_bytes_per_key(m: int, tile: int) -> float:
    """Extra H/G traffic of the 3-kernel form, bytes per key."""
    return 16.0 * m / tile
