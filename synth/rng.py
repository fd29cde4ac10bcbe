"""Counter-based random numbers (splitmix64) in torch int64.

Every draw is a pure function of (seed, stream, index), so the same graph is
produced on the CPU and on a GPU, and chunked generation gives the same bits
as one-shot generation.  torch has no uint64 arithmetic, so the 64-bit words
live in int64 tensors: multiplication wraps (two's complement), and logical
right shifts are arithmetic shifts followed by a mask.
"""
import torch

_M64 = (1 << 64) - 1
_GAMMA = 0x9E3779B97F4A7C15
_C1 = 0xBF58476D1CE4E5B9
_C2 = 0x94D049BB133111EB


def _s64(x: int) -> int:
    """Python int in [0, 2^64) -> the int64 with the same bits."""
    x &= _M64
    return x - (1 << 64) if x >= (1 << 63) else x


def splitmix64_py(x: int) -> int:
    """Reference scalar splitmix64 finaliser on Python ints (unsigned result)."""
    z = (x + _GAMMA) & _M64
    z = ((z ^ (z >> 30)) * _C1) & _M64
    z = ((z ^ (z >> 27)) * _C2) & _M64
    return z ^ (z >> 31)


def _srl(z: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (z >> k) & ((1 << (64 - k)) - 1)


def _mix(z: torch.Tensor) -> torch.Tensor:
    z = (z ^ _srl(z, 30)) * _s64(_C1)
    z = (z ^ _srl(z, 27)) * _s64(_C2)
    return z ^ _srl(z, 31)


def stream_base(seed: int, stream: int) -> int:
    """Per-(seed, stream) 64-bit offset (int64 bit pattern)."""
    return _s64(splitmix64_py(splitmix64_py(seed & _M64) ^ (stream * 0x632BE59BD9B4E019)))


def hash_u64(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """splitmix64(base(seed, stream) + idx * GAMMA) as int64 bit patterns.

    idx: int64 tensor of counters (any device).  This equals the splitmix64
    output sequence started at base, element idx.
    """
    base = stream_base(seed, stream)
    z = idx.to(torch.int64) * _s64(_GAMMA) + base
    z = z + _s64(_GAMMA)
    return _mix(z)


def hash_u64_py(seed: int, stream: int, idx: int) -> int:
    """Scalar twin of hash_u64 (unsigned result), for tests."""
    base = stream_base(seed, stream) & _M64
    return splitmix64_py((base + idx * _GAMMA) & _M64)


def uniform_int31(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """Uniform integers in [0, 2^31) (int64 tensor)."""
    return _srl(hash_u64(seed, stream, idx), 33)


def uniform_f64(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """Uniform float64 in [0, 1) with 53 random bits (exact on CPU and GPU)."""
    return _srl(hash_u64(seed, stream, idx), 11).to(torch.float64) * (2.0 ** -53)


def below(seed: int, stream: int, idx: torch.Tensor, bound: int) -> torch.Tensor:
    """Integers in [0, bound) (slight modulo bias, irrelevant here)."""
    return _srl(hash_u64(seed, stream, idx), 1) % bound


def bernoulli(seed: int, stream: int, idx: torch.Tensor, p: float) -> torch.Tensor:
    """Boolean draws with probability p, decided on 53 integer bits."""
    thr = int(p * (1 << 53))
    return _srl(hash_u64(seed, stream, idx), 11) < thr
