"""B200-native Multigrain compound sparse attention forward (Python binding of include/mg.h).

Paper: Li, Choi & Ahn, "A Slice and Dice Approach to Accelerate Compound Sparse Attention on
GPU" (IISWC 2022). The binding only marshals arguments into the C ABI of ``libmg.so``; every
step of the attention path runs in the library's sm_100a kernels. PyTorch is used for device
memory and streams only. There is no CPU fallback: a missing ``libmg.so`` raises.

    import paper_conf_iiswc_lica22_b200 as mg
    plan = mg.Plan(L=4096, heads=12, d=64, window=512, global_idx=range(32))
    O = mg.sparse_attention_fwd(plan, Q, K, V)        # Q/K/V: [B, H, L, 64] bf16 CUDA tensors
"""
from .api import (BatchedPlan, Plan, autotune_plan, selftest_umma, sparse_attention_fwd, sparse_attention_fwd_host, sparse_attention_fwd_staged,
                  sparse_attention_fwd_padded,
                  staged_buffers, staged_sddmm, staged_sizes, staged_softmax, staged_spmm, tensor_desc)
from ._lib import MGError, load as load_library, LIB_PATH, EXPORTED

__all__ = ["BatchedPlan", "Plan", "autotune_plan", "sparse_attention_fwd", "sparse_attention_fwd_host", "selftest_umma", "tensor_desc",
           "sparse_attention_fwd_staged", "sparse_attention_fwd_padded", "staged_buffers", "staged_sddmm", "staged_sizes", "staged_softmax",
           "staged_spmm",
           "MGError", "load_library", "LIB_PATH", "EXPORTED"]
