"""Pins the oracle's MurmurHash3_x64_128 (ref [1] P:276) to published values."""
import os
import struct

import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden", "murmur3_vectors.txt")


def _vectors():
    ver, texts = None, []
    for line in open(GOLD):
        line = line.rstrip("\n")
        if not line or line.startswith("#"):
            continue
        parts = line.split(" ", 3)
        if parts[0] == "verification":
            ver = int(parts[1], 16)
        elif parts[0] == "text":
            seed, hexd = int(parts[1]), parts[2]
            msg = parts[3] if len(parts) > 3 else ""
            texts.append((msg.encode(), seed, hexd))
    return ver, texts


def test_smhasher_verification_value(oracle_mod):
    ver, _ = _vectors()
    key = bytes(range(256))
    hashes = b"".join(oracle_mod.mmh3(key[:i], 256 - i) for i in range(256))
    final = oracle_mod.mmh3(hashes, 0)
    assert struct.unpack("<I", final[:4])[0] == ver == 0x6384BA69


def test_published_vectors(oracle_mod):
    _, texts = _vectors()
    assert texts
    for msg, seed, hexd in texts:
        assert oracle_mod.mmh3(msg, seed).hex() == hexd


@pytest.mark.parametrize("n", list(range(0, 40)))
def test_tail_lengths_distinct_and_stable(oracle_mod, n):
    # every tail length 0..15 and body+tail combination gives a different digest,
    # and appending a zero byte changes the digest (the length is mixed in)
    data = bytes((7 * i + 3) & 0xFF for i in range(n))
    d = oracle_mod.mmh3(data)
    assert len(d) == 16
    assert oracle_mod.mmh3(data + b"\0") != d
    assert oracle_mod.mmh3(data) == d
