"""Bullet co-run hot path on B200 (sm_100a): prefill and decode of one
transformer layer step on disjoint SM partitions of one GPU (PAPER.md
P:L7).  The compute lives in libbullet.so (csrc/, C ABI in
include/bullet.h); this package is its thin ctypes binding."""
from .bullet import (Batch, Bullet, BulletError, Model, PerfModel, CORUN, TIMESLICED, UNGATED, SMID_LOG, PROFILE, UNFUSED, UNFUSED_NORM, DEVICE_SPLIT, CHECK_KV,
                     KERNEL_KINDS,
                     EPI_F32, EPI_RESID, EPI_SILU, lib, nccl_unique_id, declared_symbols)

__all__ = ["Batch", "Bullet", "BulletError", "Model", "PerfModel", "CORUN", "TIMESLICED", "UNGATED", "SMID_LOG", "PROFILE", "UNFUSED", "UNFUSED_NORM", "DEVICE_SPLIT", "CHECK_KV", "KERNEL_KINDS",
           "EPI_F32", "EPI_RESID", "EPI_SILU", "lib", "nccl_unique_id", "declared_symbols"]
