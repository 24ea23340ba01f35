"""Python-side handle of a libsplitcnn plan (host geometry cached for buffer allocation)."""
from __future__ import annotations

from . import splitcnn as sc


class SplitPlan:
    """Owns a ``splitcnn_plan_t``.  ``O_h``/``O_w`` partition the LAST layer's output (R4)."""

    def __init__(self, layers: list[dict], N: int, C: int, H: int, W: int, O_h: list[int], O_w: list[int]):
        self.layer_dicts = layers
        self.handle = sc.splitcnn_plan_create(layers, N, C, H, W, O_h, O_w)
        self.nlayers = sc.splitcnn_plan_num_layers(self.handle)
        self.levels = [sc.splitcnn_plan_level(self.handle, m) for m in range(self.nlayers + 1)]
        self.layers = [sc.splitcnn_plan_layer(self.handle, m) for m in range(self.nlayers)]

    def __del__(self):
        h = getattr(self, "handle", None)
        if h and sc is not None and getattr(sc, "splitcnn_plan_destroy", None) is not None:
            try:
                sc.splitcnn_plan_destroy(h)
            except Exception:   # interpreter teardown
                pass
            self.handle = None

    @property
    def npatch(self) -> int:
        lv = self.levels[0]
        return lv["n_h"] * lv["n_w"]

    def level_elems(self, m: int) -> int:
        return self.levels[m]["total_elems"]

    def patch_slices(self, m: int):
        """[(i, j, offset, (N, Hp, Wp, Cpad))] of every patch buffer at level m (row-major)."""
        lv = self.levels[m]
        N, Cp, W = lv["N"], lv["Cpad"], lv["W"]
        out = []
        for i in range(lv["n_h"]):
            hp = lv["bh"][i + 1] - lv["bh"][i]
            for j in range(lv["n_w"]):
                wp = lv["bw"][j + 1] - lv["bw"][j]
                off = N * Cp * (lv["bh"][i] * W + hp * lv["bw"][j])
                out.append((i, j, off, (N, hp, wp, Cp)))
        return out

    def workspace_size(self, layer: int, dtype: int, op: int) -> int:
        return sc.splitcnn_workspace_size(self.handle, layer, dtype, op)
