"""tcgen05 operand-layout checks on the B200 (through the C ABI's mg_selftest_umma).

These pin the exact descriptor/TMEM conventions the coarse kernel relies on, against a plain
PyTorch fp32 matmul of the same bf16 operands.
"""
import pytest
import torch

import paper_conf_iiswc_lica22_b200 as mg

pytestmark = pytest.mark.gpu


def test_umma_ss_kmajor_sw128():
    g = torch.Generator().manual_seed(0)
    A = torch.randn(128, 64, generator=g).to(torch.bfloat16).cuda()
    B = torch.randn(128, 64, generator=g).to(torch.bfloat16).cuda()
    D = torch.zeros(128, 128, dtype=torch.float32, device="cuda")
    mg.selftest_umma(0, A, B, D)
    torch.cuda.synchronize()
    ref = A.float() @ B.float().T
    assert (D - ref).abs().max().item() < 1e-3


def test_umma_ts_tmem_a_mn_major_b():
    g = torch.Generator().manual_seed(1)
    A = torch.randn(128, 128, generator=g).to(torch.bfloat16).cuda()
    B = torch.randn(128, 64, generator=g).to(torch.bfloat16).cuda()
    D = torch.zeros(128, 64, dtype=torch.float32, device="cuda")
    mg.selftest_umma(1, A, B, D)
    torch.cuda.synchronize()
    ref = A.float() @ B.float()
    assert (D - ref).abs().max().item() < 1e-3
