"""Shared helpers of the GPU parity tests (test infrastructure)."""
import numpy as np
import torch

import oracle
import synth
import paper_conf_sc_cui0czlzsmylg21_b200 as ab

EPS = {ab.ABACUS_FP32: 1e-4, ab.ABACUS_BF16: 1e-2, ab.ABACUS_FP16: 1e-2}
NAMES = {ab.ABACUS_FP32: "fp32", ab.ABACUS_BF16: "bf16", ab.ABACUS_FP16: "fp16"}


_STREAM = None


def stream():
    """One explicit non-default stream for all GPU tests (the ABI maps a NULL
    stream to the ctx's own stream, which is not ordered with torch's legacy
    default stream)."""
    global _STREAM
    if _STREAM is None:
        _STREAM = torch.cuda.Stream()
        torch.cuda.set_stream(_STREAM)
    return _STREAM


class Ctx:
    def __init__(self, ops=None, params=None, precision=ab.ABACUS_FP32):
        self.ops = list(synth.OPS_PER_MODEL) if ops is None else list(ops)
        self.h = ab.abacus_create(0, self.ops)
        ab.abacus_set_stream(self.h, stream())
        if params is not None:
            self.load(params, precision)

    def load(self, params, precision):
        self.params = np.asarray(params, dtype=np.float32)
        self.precision = precision
        ab.abacus_load_predictor(self.h, self.params, precision)

    def close(self):
        ab.abacus_destroy(self.h)

    @property
    def D(self):
        return len(self.ops) + 16

    def encode(self, slots, first, count):
        x = torch.full((max(count, 1), self.D), -7, dtype=torch.int16, device="cuda")
        ab.abacus_encode_candidates(self.h, ab.make_grid(slots), first, count, x,
                                    stream())
        torch.cuda.synchronize()
        return x[:count].cpu().numpy()

    def predict(self, X):
        x = torch.from_numpy(np.ascontiguousarray(X, dtype=np.int16)).cuda()
        y = torch.full((max(len(X), 1),), float("nan"), dtype=torch.float32, device="cuda")
        ab.abacus_predict_batch(self.h, x, len(X), y, stream())
        torch.cuda.synchronize()
        return y[:len(X)].cpu().numpy().astype(np.float64)

    def encode_groups(self, groups):
        raw = ab.make_groups(groups)
        g = torch.frombuffer(bytearray(raw), dtype=torch.uint8).cuda()
        x = torch.full((max(len(groups), 1), self.D), -7, dtype=torch.int16, device="cuda")
        bad = torch.zeros(1, dtype=torch.int32, device="cuda")
        ab.abacus_encode_groups(self.h, g, len(groups), x, bad, stream())
        torch.cuda.synchronize()
        return x[:len(groups)].cpu().numpy(), int(bad.item())

    def select(self, slots, first, y, H, init=0):
        lat = torch.from_numpy(np.ascontiguousarray(y, dtype=np.float32)).cuda()
        best = torch.tensor([init], dtype=torch.int64, device="cuda")
        ab.abacus_select_group(self.h, ab.make_grid(slots), first, len(y), lat, H, best,
                               stream())
        torch.cuda.synchronize()
        return int(best.item()) & (2**64 - 1)


def rel_err(y, ref, floor=None):
    d = np.abs(np.asarray(ref, dtype=np.float64))
    if floor is not None:
        d = np.maximum(d, floor)
    return np.abs(np.asarray(y, dtype=np.float64) - ref) / d


def accept_key(gpu_key, strict, loose):
    """Reading c18: several answers are correct near the threshold."""
    return strict <= gpu_key <= loose
