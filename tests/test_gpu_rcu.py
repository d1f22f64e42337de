"""GPU parity of the f3 path (SRCU + RCU delegation, ga_rcu_list_removal)
against the oracle (oracle/rcu.py): the Fig. 6 benchmark's outcome is unique
-- every list element whose tag is in the input is removed exactly once, the
list ends empty -- and the grace-period property is observable: no reader
reaches an element after its release (the kernel counts violations), no
element is released twice.  Sizes span small lists, many warps per writer and
more threads than the GPU holds at once."""
import numpy as np
import pytest
import torch

import tracegen
from oracle import rcu as orcu

pytestmark = pytest.mark.gpu

ga = pytest.importorskip("paper_conf_ppopp_geladog19_b200")


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    torch.cuda.set_device(0)


@pytest.mark.timeout(600, method="thread")
@pytest.mark.parametrize("T,ratio", [(64, 32), (1000, 32), (4096, 128), (32768, 32), (65536, 2048),
                                     (400000, 512)])
@pytest.mark.parametrize("delegate", [0, 1])
def test_list_removal_matches_oracle(T, ratio, delegate):
    W = max(1, T // ratio)
    tags_np = tracegen.rcu_tags(T, W)
    removed, live = orcu.list_removal(range(W), tags_np.tolist())
    tags = torch.from_numpy(tags_np.view(np.int32)).cuda()
    wsb = ga.ga_rcu_workspace_bytes(W)
    ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    out = torch.zeros(8, dtype=torch.int64, device="cuda")
    ga.ga_rcu_list_removal(torch.cuda.current_stream().cuda_stream, T, W, tags.data_ptr(), ws.data_ptr(), wsb,
                           delegate, 256, out.data_ptr())
    torch.cuda.synchronize()
    o = [int(x) for x in out.cpu().numpy()]
    assert o[0] == len(removed) == W            # every list element unlinked once
    assert o[1] == W                            # every release callback ran once
    assert o[5] == 0                            # no double release
    assert o[6] == len(live) == 0               # the list is empty
    assert o[7] == T - W                        # everyone else was a reader
    assert o[2] == 0                            # no reader reached a released element
    if delegate:
        assert o[3] + o[4] == W                 # each writer ran a barrier or delegated it
    else:
        assert o[3] == W and o[4] == 0


def test_workspace_size_and_bad_arguments():
    assert ga.ga_rcu_workspace_bytes(1) > 0
    with pytest.raises(Exception):
        ga.ga_rcu_workspace_bytes(0)
