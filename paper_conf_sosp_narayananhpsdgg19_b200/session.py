"""Pipeline session: wires the C-ABI calls together for one process (all workers local,
several "virtual" workers may share a GPU) or one process per GPU (torch.distributed
exchanges the CUDA-IPC blobs; plumbing only, no data-path collective)."""
from __future__ import annotations

import struct
from typing import Callable, Dict, List, Optional, Sequence

import numpy as np

from . import (PD_BF16, PD_SGD, Plan, pd_create, pd_destroy, pd_export_worker, pd_get_layer_times, pd_get_losses,
               pd_get_params, pd_get_stats, pd_get_trace, pd_get_version_map, pd_import_worker, pd_set_data,
               pd_set_layer_profiling, pd_set_timing, pd_stage_init, pd_stage_solo, pd_run, pd_save_checkpoint,
               pd_load_checkpoint)


def workers_of(plan: Plan):
    """(worker id, stage, replica, gpu) in plan order (consecutive GPUs per stage, R18)."""
    out, wid = [], 0
    for s, (first, last, reps, gpu0) in enumerate(plan.stages):
        for r in range(reps):
            out.append((wid, s, r, gpu0 + r))
            wid += 1
    return out


def blob_worker(blob: bytes):
    """(stage, replica) a pd_export_worker blob describes."""
    _magic, stage, replica = struct.unpack_from("<Iii", blob, 0)
    return stage, replica


def stage_of_rank(plan: Plan, rank: int) -> int:
    """Stage whose replica runs on process `rank` (one process per GPU, R18 placement)."""
    for s, (first, last, reps, gpu0) in enumerate(plan.stages):
        if gpu0 <= rank < gpu0 + reps:
            return s
    raise ValueError(f"rank {rank} is outside the plan's {sum(st[2] for st in plan.stages)} GPUs")


class Pipeline:
    def __init__(self, plan: Plan, layers, params: Sequence[np.ndarray], *, dtype=PD_BF16, optimizer=PD_SGD,
                 lr=0.01, beta1=0.9, beta2=0.999, eps=1e-8, minibatch=1, record_trace=1, max_depth=0,
                 sync_mode=0, device_of: Optional[Callable[[int], int]] = None, local: Optional[Callable[[int], bool]] = None,
                 allgather: Optional[Callable[[list], list]] = None, solo: bool = False):
        """device_of(worker_gpu) -> CUDA ordinal (default: everything on device 0, i.e. virtual
        workers); local(worker_id) -> whether this process owns the worker (default all);
        allgather(list_of_bytes) -> list over processes of lists (needed when not all local);
        solo: measure the local workers alone (pd_stage_solo) instead of importing peers."""
        self.plan, self.layers = plan, list(layers)
        self.ctx = pd_create(plan, self.layers, dtype, optimizer, lr, beta1, beta2, eps, minibatch, record_trace,
                             max_depth, sync_mode)
        device_of = device_of or (lambda g: 0)
        local = local or (lambda w: True)
        self.workers = workers_of(plan)
        self.local_ids = [w for w, s, r, g in self.workers if local(w)]
        for wid, s, r, g in self.workers:
            if not local(wid):
                continue
            first, last = plan.stages[s][0], plan.stages[s][1]
            pd_stage_init(self.ctx, s, r, device_of(g), [params[l] for l in range(first, last + 1)])
        if solo:
            pd_stage_solo(self.ctx)
        elif len(self.local_ids) < len(self.workers):
            if allgather is None:
                raise ValueError("remote workers need an allgather for the IPC blobs")
            mine = [pd_export_worker(self.ctx, s, r) for wid, s, r, g in self.workers if local(wid)]
            local_sr = {(s, r) for wid, s, r, g in self.workers if local(wid)}
            for blobs in allgather(mine):
                for b in blobs:
                    # our own blobs come back too: skip them by (stage, replica) (blob header
                    # {u32 magic, i32 stage, i32 replica, ...}, include/pipedream.h); every other
                    # import error is real and propagates
                    if blob_worker(b) in local_sr:
                        continue
                    pd_import_worker(self.ctx, b)

    def save_checkpoint(self, directory):
        pd_save_checkpoint(self.ctx, directory)

    def load_checkpoint(self, directory):
        pd_load_checkpoint(self.ctx, directory)

    def set_data(self, inputs, tokens, labels, n):
        pd_set_data(self.ctx, inputs, tokens, labels, n)

    def run(self, M, noam=0):
        pd_run(self.ctx, M, noam)

    def params(self, layer_sizes: Sequence[int], layers: Optional[Sequence[int]] = None) -> Dict[int, np.ndarray]:
        layers = range(len(self.layers)) if layers is None else layers
        return {l: pd_get_params(self.ctx, l, layer_sizes[l]) for l in layers}

    def trace(self):
        return pd_get_trace(self.ctx)

    def version_map(self, M):
        return pd_get_version_map(self.ctx, len(self.plan.stages), M)

    def losses(self, M):
        return pd_get_losses(self.ctx, M)

    def stats(self):
        return pd_get_stats(self.ctx)

    def set_timing(self, record_trace, kernel_timing_mask=0xFF):
        pd_set_timing(self.ctx, record_trace, kernel_timing_mask)

    def set_layer_profiling(self, on: bool):
        pd_set_layer_profiling(self.ctx, on)

    def layer_times(self):
        """(forward s, backward s) per layer, mean per minibatch of the last run."""
        return pd_get_layer_times(self.ctx, len(self.layers))

    def close(self):
        if self.ctx is not None:
            pd_destroy(self.ctx)
            self.ctx = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def torch_allgather(group=None):
    """allgather over torch.distributed (gloo or nccl), for Pipeline(allgather=...)."""
    import torch.distributed as dist

    def ag(obj):
        out = [None] * dist.get_world_size(group)
        dist.all_gather_object(out, obj, group=group)
        return out

    return ag
