"""Counter-based 64-bit generator (SplitMix64 finaliser), implemented twice with
bit-identical results: numpy (uint64, host) and torch (int64, any device).

value(seed, stream, i) = mix(mix(seed ^ (stream * K1)) + (i + 1) * GOLDEN)

Large graphs (RMAT scale 22/26) are generated with the torch version on the GPU;
small ones with numpy.  ``tests/test_inputs.py`` checks the two agree.
"""
import numpy as np

GOLDEN = 0x9E3779B97F4A7C15
K1 = 0xD1B54A32D192ED03
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB
_U64 = (1 << 64) - 1


def _signed(x):
    """uint64 constant -> the int64 with the same bit pattern (for torch)."""
    x &= _U64
    return x - (1 << 64) if x >= (1 << 63) else x


def splitmix64_np(z):
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + np.uint64(GOLDEN)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(M1)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(M2)
        z = z ^ (z >> np.uint64(31))
    return z


def _key(seed, stream):
    s = ((seed & _U64) ^ ((stream * K1) & _U64)) & _U64
    return int(splitmix64_np(np.uint64(s)))


def counter_u64_np(seed, stream, start, count):
    """uint64 array of values i = start .. start+count-1."""
    key = np.uint64(_key(seed, stream))
    i = np.arange(start + 1, start + count + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = key + i * np.uint64(GOLDEN)
    return splitmix64_np(x)


def _srl(z, s):
    """logical right shift of an int64 tensor (torch's >> is arithmetic)."""
    return (z >> s) & ((1 << (64 - s)) - 1)


def counter_u64_torch(seed, stream, start, count, device="cpu"):
    """int64 tensor with the same bit patterns as ``counter_u64_np``."""
    import torch
    key = _signed(_key(seed, stream))
    i = torch.arange(start + 1, start + count + 1, dtype=torch.int64, device=device)
    x = i * _signed(GOLDEN) + key
    z = x + _signed(GOLDEN)
    z = (z ^ _srl(z, 30)) * _signed(M1)
    z = (z ^ _srl(z, 27)) * _signed(M2)
    z = z ^ _srl(z, 31)
    return z
