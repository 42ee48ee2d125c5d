"""Caller-owned arena (lt_config.arena; "caller-owned device memory (torch tensor) ... the
library sub-allocates all pools from it once"): every pool of a run comes out of the caller's tensor, the
paths stay bit-exact, a graph load starts the arena over, exhaustion is LT_ERR_OOM, and the device
memory outside the arena does not move."""
import numpy as np
import pytest

import lt_inputs
import oracle as O
import paper_conf_icde_xing0wxl23_b200 as LT

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def g13():
    return lt_inputs.rmat_cpu(13, 8 * 2 ** 13, seed=3)


@pytest.mark.parametrize("P,layout", [(1, LT.LAYOUT_ADJ), (4, LT.LAYOUT_CSR), (8, LT.LAYOUT_ADJ12)])
def test_arena_holds_every_pool(gpu, g13, P, layout):
    import torch
    arena = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    free0, _ = torch.cuda.mem_get_info()
    starts = lt_inputs.deepwalk_starts(3 * g13.n, g13.n)
    with LT.Engine(arena=arena, layout=layout, chunk_walks=512, visit_counts=True) as e:
        e.graph_load(g13.row_ptr, g13.col, P)
        for seed in (1, 2):
            e.walks_init(starts, LT.DEEPWALK, 12, seed)
            e.run()
            paths, lengths = e.get_paths()
            op, ol, _, _ = O.walks(g13.row_ptr, g13.col, starts, app=O.DEEPWALK, length=12, seed=seed)
            np.testing.assert_array_equal(lengths, ol)
            np.testing.assert_array_equal(paths, op)
        used = e.stats()["arena_bytes_used"]
        torch.cuda.synchronize()
        free1, _ = torch.cuda.mem_get_info()
        # a second graph load starts the arena over (same footprint), PPR on it
        e.graph_load(g13.row_ptr, g13.col, P)
        ps = lt_inputs.ppr_starts(10_000, g13.argmax_deg)
        e.walks_init(ps, LT.PPR, 0.15, 3)
        e.run()
        paths, lengths = e.get_paths()
        op, ol, _, _ = O.walks(g13.row_ptr, g13.col, ps, app=O.PPR, alpha=0.15, seed=3)
        np.testing.assert_array_equal(paths, op)
        assert e.stats()["arena_bytes_used"] <= used + (8 << 20)
    assert 0 < used <= arena.numel()
    assert free0 - free1 < (16 << 20), (free0 - free1)  # the pools live in the arena, not in new allocations


def test_arena_exhaustion_is_oom(gpu, g13):
    import torch
    arena = torch.empty(64 << 10, dtype=torch.uint8, device="cuda")
    with LT.Engine(arena=arena) as e:
        with pytest.raises(LT.LTError) as ex:
            e.graph_load(g13.row_ptr, g13.col, 4)
        assert ex.value.status == LT.LT_ERR_OOM


def test_arena_rejects_ipc_path_matrix(gpu, g13):
    import torch
    arena = torch.empty(64 << 20, dtype=torch.uint8, device="cuda")
    with LT.Engine(arena=arena, rank=0, world=2) as e:
        e.graph_load(g13.row_ptr, g13.col, 2)
        e.walks_init(lt_inputs.deepwalk_starts(100, g13.n), LT.DEEPWALK, 5, 1)
        with pytest.raises(LT.LTError):
            e.paths_buffers()
    with pytest.raises(ValueError):
        LT.Engine(arena=np.zeros(4096, np.uint8))
