"""CPU checks of the C-ABI library: it loads, exports every symbol include/lt.h declares, its host
partitioner is right, and it fails cleanly (status codes, no crash) without a GPU."""
import ctypes
import os
import re

import numpy as np
import pytest

import lt_inputs
import paper_conf_icde_xing0wxl23_b200 as LT
from paper_conf_icde_xing0wxl23_b200 import lt as ltmod

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "lt.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lt_[a-z0-9_]+)\s*\(", src)))


def test_exports_every_declared_symbol():
    names = _declared()
    assert len(names) >= 15
    lib = ctypes.CDLL(ltmod.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(ltmod.EXPORTED) == names


def test_product_never_touches_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icde_xing0wxl23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                s = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in s and "from oracle" not in s and "oracle.h" not in s, f


def _brute_bounds(row_ptr, P):
    n = len(row_ptr) - 1
    cost = 8 * np.arange(n + 1, dtype=object) + 4 * np.asarray(row_ptr, dtype=object)
    b = [0]
    for k in range(1, P):
        target = (cost[n] * k) // P if (cost[n] * k) % P == 0 else None
        # lower_bound of the exact rational k*cost(n)/P
        v = next(v for v in range(n + 1) if cost[v] * P >= cost[n] * k)
        b.append(v)
    b.append(n)
    for k in range(1, P):
        b[k] = max(b[k], b[k - 1] + 1)
    for k in range(P - 1, 0, -1):
        b[k] = min(b[k], b[k + 1] - 1)
    return np.array(b, dtype=np.uint32)


@pytest.mark.parametrize("P", [1, 2, 3, 4, 7, 16, 100])
def test_partition_bounds_brute_force(P):
    g = lt_inputs.rmat_cpu(9, 4000, seed=2)
    b = LT.partition_bounds(g.row_ptr, P)
    np.testing.assert_array_equal(b, _brute_bounds(g.row_ptr, P))
    assert b[0] == 0 and b[-1] == g.n and np.all(np.diff(b.astype(np.int64)) >= 1)


def test_partition_bounds_degenerate():
    g = lt_inputs.small_graph([(0, 1), (1, 2), (2, 3)])
    np.testing.assert_array_equal(LT.partition_bounds(g.row_ptr, 4), [0, 1, 2, 3, 4])   # P == n
    # one huge vertex: bounds still strictly increasing
    g = lt_inputs.small_graph([(0, k) for k in range(1, 50)])
    b = LT.partition_bounds(g.row_ptr, 8)
    assert np.all(np.diff(b.astype(np.int64)) >= 1) and b[-1] == 50
    with pytest.raises(LT.LTError):
        LT.partition_bounds(g.row_ptr, 0)
    with pytest.raises(LT.LTError):
        LT.partition_bounds(g.row_ptr, 51)


def test_partition_bounds_balance_bytes():
    g = lt_inputs.rmat_cpu(14, 16 * 2 ** 14, seed=1)
    P = 16
    b = LT.partition_bounds(g.row_ptr, P).astype(np.int64)
    rp = g.row_ptr.astype(np.int64)
    cost = 8 * b + 4 * rp[b]
    part = np.diff(cost)
    maxdeg_bytes = 8 + 4 * g.max_deg
    assert part.max() - part.min() <= 2 * maxdeg_bytes + 16


@pytest.mark.skipif(os.environ.get("CUDA_VISIBLE_DEVICES", None) is None and __import__("torch").cuda.is_available(),
                    reason="GPU present: covered by gpu tests")
def test_create_without_gpu_fails_cleanly():
    with pytest.raises(LT.LTError) as ei:
        LT.Engine()
    assert ei.value.status in (ltmod.LT_ERR_CUDA, ltmod.LT_ERR_INVALID)


def test_struct_layout_matches_header(tmp_path):
    """The ctypes mirrors of lt_config / lt_stats / lt_pool_state match the C compiler's layout."""
    import subprocess
    src = tmp_path / "sz.c"
    src.write_text('#include <stdio.h>\n#include <stddef.h>\n#include "lt.h"\nint main(){printf("%zu %zu %zu %zu %zu\\n",'
                   ' sizeof(lt_config), sizeof(lt_stats), sizeof(lt_pool_state), offsetof(lt_config, graph_pool_bytes),'
                   ' offsetof(lt_stats, iterations));}\n')
    exe = tmp_path / "sz"
    subprocess.run(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)], check=True)
    sizes = [int(x) for x in subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split()]
    assert sizes == [ctypes.sizeof(ltmod.Config), ctypes.sizeof(ltmod.Stats), ctypes.sizeof(ltmod.PoolState),
                     ltmod.Config.graph_pool_bytes.offset, ltmod.Stats.iterations.offset]


# ---- compressed partition format (lt_config.ooc_compress): the host encoder against an independent decoder
def _decode_blocks(hdr, pay, n):
    """Decode the documented format (include/lt.h, lt_compress_columns) with plain integer arithmetic."""
    out = np.zeros(n, dtype=np.uint64)
    pay = [int(x) for x in pay]
    for j in range((n + 31) // 32):
        base, off = int(hdr[j, 0]), int(hdr[j, 1])
        w = int(hdr[j + 1, 1]) - off
        acc = base
        for i in range(min(32, n - 32 * j)):
            z = 0
            if i and w:
                bit = i * w
                word = pay[off + (bit >> 5)] | ((pay[off + (bit >> 5) + 1] << 32) if (bit & 31) + w > 32 else 0)
                z = (word >> (bit & 31)) & ((1 << w) - 1)
            delta = (z >> 1) ^ (-(z & 1) & 0xFFFFFFFF)  # unzigzag, mod 2^32
            acc = (acc + delta) & 0xFFFFFFFF if i else base
            out[32 * j + i] = acc
    return out


@pytest.mark.parametrize("kind", ["sorted_rmat", "random_u32", "extremes", "constant", "short"])
def test_compress_columns_roundtrip(kind):
    rng = np.random.default_rng(11)
    if kind == "sorted_rmat":
        g = lt_inputs.rmat_cpu(12, 65_536, seed=1)
        col = g.col.astype(np.uint32)
    elif kind == "random_u32":
        col = rng.integers(0, 1 << 32, 1000, dtype=np.uint64).astype(np.uint32)  # differences >= 2^31: w = 32
    elif kind == "extremes":
        col = np.where(np.arange(777) % 3 == 0, 0, 0xFFFFFFFF).astype(np.uint32)
    elif kind == "constant":
        col = np.full(100, 12345, dtype=np.uint32)  # width 0: no payload
    else:
        col = np.array([7, 3], dtype=np.uint32)
    hdr, pay = LT.compress_columns(col)
    assert hdr.shape == ((len(col) + 31) // 32 + 1, 2)
    np.testing.assert_array_equal(_decode_blocks(hdr, pay, len(col)), col.astype(np.uint64))
    widths = np.diff(hdr[:, 1].astype(np.int64))
    assert widths.min() >= 0 and widths.max() <= 32
    if kind == "sorted_rmat":  # sorted adjacency compresses: fewer bytes than 4 per entry
        assert 8 * len(hdr) + 4 * len(pay) < 4 * len(col)
    if kind == "random_u32":
        assert widths.max() == 32
    if kind == "constant":
        assert len(pay) == 0
