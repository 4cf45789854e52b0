"""GPU: dslash_timeline (DSLASH_OPT_TIMING) records the halo exchange on the communication stream
next to the stencil kernels, on one clock, and kernel_timing(ALL) still counts kernels only."""
import pytest

import fieldgen

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("kw", [{}, {"self_nccl": True}, {"transport": "p2p"}])
def test_timeline_records_exchange_and_kernels(kw):
    import torch
    from paper_conf_sc_dufekgaad024_b200 import Dslash, _abi
    torch.cuda.set_device(0)
    dims = (8, 8, 8, 12)
    fat, lng = fieldgen.workload_links(dims)
    src = torch.from_numpy(fieldgen.vector_cb(dims, 3, 1)).cuda()
    with Dslash(dims, parity_mask=0, force_halo=0x8, timing=True, **kw) as D:
        D.load_links(fat, lng)
        out = D.empty_vector()
        for _ in range(3):
            D.apply(out, src, 0)
        torch.cuda.synchronize()
        tl = D.timeline()
        kinds = [k for k, _, _ in tl]
        assert kinds.count("exchange") == 3 and kinds.count("interior") == 3 and kinds.count("boundary") == 3
        assert tl[0][1] == 0.0 and all(b >= a >= 0.0 for _, a, b in tl)
        # per apply: the boundary kernel cannot start before its exchange started
        ex = [(a, b) for k, a, b in tl if k == "exchange"]
        bd = [(a, b) for k, a, b in tl if k == "boundary"]
        assert all(b[0] >= e[0] for e, b in zip(ex, bd))
        tot, n = D.kernel_timing(_abi.DSLASH_TIMING_ALL)
        assert n == 6                                     # interior + boundary per apply, no exchanges
        xt, xn = D.kernel_timing(_abi.DSLASH_TIMING_EXCHANGE)
        assert xn == 3 and xt > 0
        D.kernel_timing_reset()
        assert D.timeline() == []
