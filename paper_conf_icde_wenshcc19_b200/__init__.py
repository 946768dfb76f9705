"""GMP-SVM hot path on B200 (sm_100a): batched RBF kernel values shared across the one-vs-one
pairs, batched working-set SMO, Platt sigmoids, shared-SV decision values and pairwise
coupling -- behind the C ABI of include/gmpsvm.h (libgmpsvm.so).

Paper: Wen et al., "Efficient Multi-Class Probabilistic SVMs on GPUs", ICDE 2019.
"""
from ._lib import (EFORMAT, EINVAL, ENOMEM, ENOTIMPL, ECUDA, OK, WARN_MAXITER, GmpsvmError, Model, Shard, couple,
                   last_predict_stats, launch_count, lib, model_from_alpha, rbf_kernel, shard_merge, train, train_csr)

__all__ = ["train", "train_csr", "Model", "Shard", "shard_merge", "model_from_alpha", "rbf_kernel", "couple", "launch_count", "last_predict_stats", "lib", "GmpsvmError",
           "OK", "WARN_MAXITER", "EINVAL", "ENOMEM", "ECUDA", "ENOTIMPL", "EFORMAT"]
