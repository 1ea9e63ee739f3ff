"""libds calls inside CUDA graphs: the _ex forms do no host synchronisation and
allocate nothing once the stream's workspace exists, and every launch re-arms
its own ticket word (R24), so a captured call replays correctly.  Captured
here with torch.cuda.graph on its side stream, replayed on restored inputs."""
import numpy as np
import pytest
import torch

import dsgen
import oracle
from paper_conf_icpp_gomez_lunacshg15_b200 import libds

pytestmark = pytest.mark.gpu


def test_compact_pad_in_a_graph():
    n = 3 * 8192 * 17 + 5
    src = dsgen.compact_input(n, 0.4, 77, device="cuda")
    exp = src.cpu().numpy().view(np.uint32).copy()
    m = oracle.compact(exp, 0)
    R, C, NC = 300, 257, 260
    msrc = dsgen.matrix_input(R, C, NC, 4, device="cuda")
    mexp = msrc.cpu().numpy().view(np.uint32).copy()
    oracle.pad(mexp, R, C, NC, 4)
    work, mwork = torch.empty_like(src), torch.empty_like(msrc)
    d_n = torch.zeros(1, dtype=torch.int64, device="cuda")
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):  # warm-up on the capture stream: its workspace is made here
        work.copy_(src)
        libds.ds_compact_ex(work, n, 0, d_n, s)
        mwork.copy_(msrc)
        libds.ds_pad_ex(mwork, R, C, NC, 4, None, s)
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s):
        work.copy_(src)
        libds.ds_compact_ex(work, n, 0, d_n, s)
        mwork.copy_(msrc)
        libds.ds_pad_ex(mwork, R, C, NC, 4, None, s)
    for rep in range(5):
        d_n.zero_()
        work.fill_(-1)
        g.replay()
        torch.cuda.synchronize()
        assert int(d_n.item()) == m, rep
        assert np.array_equal(work.cpu().numpy().view(np.uint32), exp), rep
        assert np.array_equal(mwork.cpu().numpy().view(np.uint32), mexp), rep
