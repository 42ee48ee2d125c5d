"""SURVEY.md §4 pin P2: the device Philox4x32-10 of the update kernels (lt_philox_device) equals cuRAND's
curand_Philox4x32_10 on random counters and keys, and the walk RNG's counter layout (reading R3:
blk(w, t, 0) = Philox(ctr = {t, 0, w lo, w hi}, key = seed halves)) equals cuRAND's
curand_init(seed, subsequence w, offset 4t) + curand4(). Paths already match the CPU oracle bit-exactly,
which pins the device RNG transitively; this pins it directly against a library routine. The cuRAND side
is tests/cuda/curand_ref.cu, compiled here with nvcc."""
import ctypes
import os
import subprocess

import numpy as np
import pytest

import paper_conf_icde_xing0wxl23_b200 as LT

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def curand_ref(tmp_path_factory):
    so = str(tmp_path_factory.mktemp("curand") / "libcurand_ref.so")
    subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2", "-shared", "-Xcompiler", "-fPIC",
                    os.path.join(HERE, "cuda", "curand_ref.cu"), "-o", so], check=True)
    lib = ctypes.CDLL(so)
    lib.curand_philox_blocks.argtypes = [ctypes.c_void_p] * 3 + [ctypes.c_uint64]
    lib.curand_stream_blocks.argtypes = [ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                         ctypes.c_uint64]
    return lib


def test_device_philox_equals_curand(gpu, curand_ref):
    rng = np.random.default_rng(7)
    n = 1 << 16
    ctr = rng.integers(0, 1 << 32, size=(n, 4), dtype=np.uint64).astype(np.uint32)
    key = rng.integers(0, 1 << 32, size=(n, 2), dtype=np.uint64).astype(np.uint32)
    ctr[:3] = [[0, 0, 0, 0], [0xFFFFFFFF] * 4, [0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344]]
    key[:3] = [[0, 0], [0xFFFFFFFF] * 2, [0xA4093822, 0x299F31D0]]
    ours = LT.philox_device(ctr, key)
    ref = np.zeros_like(ctr)
    assert curand_ref.curand_philox_blocks(ctr.ctypes.data, key.ctypes.data, ref.ctypes.data, n) == 0
    np.testing.assert_array_equal(ours, ref)
    # the published known-answer vectors (Random123), also pinned on the CPU oracle (P1)
    assert ours[0].tolist() == [0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8]
    assert ours[2].tolist() == [0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1]


def test_walk_counter_layout_equals_curand_stream(gpu, curand_ref):
    """blk(w, t, 0) = Philox({t, 0, w lo, w hi}, seed halves) is cuRAND's subsequence w at offset 4t."""
    rng = np.random.default_rng(8)
    n = 1 << 14
    seed = 0x0123456789ABCDEF
    w = rng.integers(0, 1 << 40, size=n, dtype=np.uint64)
    t = rng.integers(0, 1 << 20, size=n, dtype=np.uint64).astype(np.uint32)
    ctr = np.stack([t, np.zeros(n, np.uint32), (w & 0xFFFFFFFF).astype(np.uint32), (w >> 32).astype(np.uint32)], 1)
    key = np.tile(np.array([seed & 0xFFFFFFFF, seed >> 32], dtype=np.uint32), (n, 1))
    ours = LT.philox_device(ctr, key)
    ref = np.zeros((n, 4), dtype=np.uint32)
    assert curand_ref.curand_stream_blocks(seed, w.ctypes.data, t.ctypes.data, ref.ctypes.data, n) == 0
    np.testing.assert_array_equal(ours, ref)
