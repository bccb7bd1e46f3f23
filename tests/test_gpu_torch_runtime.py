"""PyTorch integration (survey §8(f) rank 3): a real Tree-LSTM trained with torch operators while
its tensors live in libdyo-managed memory (CPU-first homes, arena slots per block, block-boundary
events, on-demand fetch of the nodes the pilot placed in the wrong order inside a block) computes
bit-identical weights to the same model with every tensor resident on the device."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import workloads as WL


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()


@pytest.mark.parametrize("budget_mib", [16, 64])
def test_offloaded_training_equals_resident(budget_mib):
    from paper_conf_hpca_renxyzlnwxl24_b200.torch_runtime import TreeLSTMRuntime
    wl = WL.make("tree", n_samples=16, batch=4, max_leaves=16, hidden=128, budget=budget_mib << 20)
    ref = TreeLSTMRuntime(wl, mode="resident")
    off = TreeLSTMRuntime(wl, mode="dyo")
    for s in range(3):
        ids = [(4 * s + i) % 16 for i in range(4)]
        ref.step(ids)
        off.step(ids)
    wr, wo = ref.weights(), off.weights()
    for k in wr:
        assert np.array_equal(wr[k], wo[k]), k
    off.close()
    assert off.faults["faults"] > 0            # leaves / internal nodes re-ordered inside blocks
