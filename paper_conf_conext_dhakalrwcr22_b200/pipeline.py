"""Torch-buffer convenience layer over the C ABI (argument marshalling only).

``OrbPipeline`` owns one ss_ctx plus torch CUDA output buffers sized for ``max_frames``:
    kps    [max_frames, kp_capacity] ss_keypoint  (as a uint8 [.., 20] tensor)
    desc   [max_frames, kp_capacity, 32] uint8
    counts [max_frames, n_levels + 1] int32
and exposes extract / match calls that enqueue on a torch stream.
"""
from __future__ import annotations

import numpy as np
import torch

from . import ss


class OrbPipeline:
    def __init__(self, width: int, height: int, n_features: int = 1000, n_levels: int = 8,
                 scale_factor: float = 1.2, ini_th: int = 20, min_th: int = 7, max_frames: int = 4,
                 max_queries: int = 0, max_map: int = 0, device: int = 0):
        if not torch.cuda.is_available():
            raise RuntimeError("OrbPipeline needs a CUDA device (no CPU fallback by design)")
        self.device = torch.device("cuda", device)
        self.params = ss.ss_orb_params_init(width, height, n_features, n_levels, scale_factor, ini_th, min_th)
        self.ctx = ss.ss_create(device, self.params, max_frames, max_queries, max_map)
        self.width, self.height = width, height
        self.n_levels = n_levels
        self.cap = self.params.kp_capacity
        self.max_frames = max_frames
        self.kps = torch.zeros((max_frames, self.cap, 20), dtype=torch.uint8, device=self.device)
        self.desc = torch.zeros((max_frames, self.cap, ss.DESC_BYTES), dtype=torch.uint8, device=self.device)
        self.counts = torch.zeros((max_frames, n_levels + 1), dtype=torch.int32, device=self.device)
        self.prepared_rows = 0

    def set_distribution(self, mode: int):
        """ss.SS_DIST_QUADTREE (default) or ss.SS_DIST_GRID_TOPN for the following extracts."""
        ss.ss_set_distribution(self.ctx, mode)

    def close(self):
        if self.ctx:
            ss.ss_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- hot path -------------------------------------------------------------------
    def extract(self, frames: torch.Tensor, stream: torch.cuda.Stream | None = None, n_frames: int | None = None):
        """frames: uint8 CUDA tensor [B, H, pitch] (row pitch = frames.stride(1))."""
        assert frames.dtype == torch.uint8 and frames.is_cuda and frames.dim() == 3
        assert frames.stride(2) == 1
        B = frames.shape[0] if n_frames is None else n_frames
        stream = stream or torch.cuda.current_stream(self.device)
        ss.ss_orb_extract(self.ctx, B, frames, frames.stride(0), frames.stride(1), self.kps, self.desc,
                          self.counts, stream)

    def match_window(self, n_frames: int, queries: torch.Tensor, qdesc: torch.Tensor, out: torch.Tensor,
                     taken: torch.Tensor | None = None, cfg: ss.ss_match_cfg | None = None,
                     stream: torch.cuda.Stream | None = None):
        cfg = cfg or ss.window_cfg()
        stream = stream or torch.cuda.current_stream(self.device)
        nq = queries.numel() // 20 if queries.dtype == torch.uint8 else queries.shape[0]
        ss.ss_match_projection(self.ctx, n_frames, self.kps, self.desc, self.counts, taken, nq, queries, qdesc,
                               0, cfg, out, stream)

    def prepare_map(self, map_desc: torch.Tensor, stream: torch.cuda.Stream | None = None):
        """ss_brute_map_prepare: expand a (static) shared map once; match_brute(n, None, out)
        then uses it."""
        stream = stream or torch.cuda.current_stream(self.device)
        ss.ss_brute_map_prepare(self.ctx, map_desc, map_desc.shape[0], stream)
        self.prepared_rows = map_desc.shape[0]

    def match_brute(self, n_frames: int, map_desc: torch.Tensor | None, out: torch.Tensor,
                    cfg: ss.ss_match_cfg | None = None, stream: torch.cuda.Stream | None = None):
        """map_desc [n_map, 32] uint8 CUDA tensor, or None for the prepared map (prepare_map)."""
        cfg = cfg or ss.brute_cfg()
        stream = stream or torch.cuda.current_stream(self.device)
        n_map = self.prepared_rows if map_desc is None else map_desc.shape[0]
        ss.ss_match_projection(self.ctx, n_frames, self.kps, self.desc, self.counts, None, 0, None, map_desc,
                               n_map, cfg, out, stream)

    def project(self, n_frames: int, cams: torch.Tensor, points: torch.Tensor, point_frame: torch.Tensor,
                out: torch.Tensor, th: float = 1.0, stream: torch.cuda.Stream | None = None):
        """O11: cams uint8 [n_frames, 96] (ss_camera), points uint8 [n, 32] (ss_map_point),
        point_frame int32 [n] -> out uint8 [n, 20] (ss_mp_query), the WINDOW queries."""
        stream = stream or torch.cuda.current_stream(self.device)
        n = point_frame.numel()
        ss.ss_project_points(self.ctx, n_frames, cams, n, points, point_frame, th, out, stream)

    def stereo(self, frames: torch.Tensor, bf: float, baseline: float, uright: torch.Tensor, depth: torch.Tensor,
               n_pairs: int | None = None, stream: torch.cuda.Stream | None = None):
        """O12 after extract(frames) of pairs (2i left, 2i+1 right): uright / depth f32 [n_pairs, cap]."""
        stream = stream or torch.cuda.current_stream(self.device)
        n_pairs = frames.shape[0] // 2 if n_pairs is None else n_pairs
        ss.ss_stereo_match(self.ctx, n_pairs, frames, frames.stride(0), frames.stride(1), self.kps, self.desc,
                           self.counts, bf, baseline, uright, depth, stream)

    def match_last_frame(self, n_frames: int, cams: torch.Tensor, point_offsets: torch.Tensor, points: torch.Tensor,
                         pdesc: torch.Tensor, out: torch.Tensor, n_matches: torch.Tensor | None = None,
                         last_cams: torch.Tensor | None = None, mb: float = 0.0, th: float = 15.0, th_high: int = 100,
                         check_orientation: bool = True, min_matches: int = 20, taken: torch.Tensor | None = None,
                         matched: torch.Tensor | None = None, stream: torch.cuda.Stream | None = None):
        """O13 after extract(): cams / last_cams uint8 [n_frames, 96] (ss_camera), point_offsets int32
        [n_frames+1], points uint8 [n, 24] (ss_frame_point), pdesc uint8 [n, 32] -> out int32 [n, 3]
        (ss_match), n_matches int32 [n_frames], matched uint8 [n_frames, cap] (taken | kept matches)."""
        stream = stream or torch.cuda.current_stream(self.device)
        ss.ss_match_last_frame(self.ctx, n_frames, cams, last_cams, mb, self.kps, self.desc, self.counts, taken,
                               point_offsets, points, pdesc, th, th_high, int(check_orientation), min_matches, out,
                               n_matches, matched, stream)

    # -- host views (synchronising; tests / examples) -------------------------------
    def results(self, n_frames: int):
        torch.cuda.synchronize(self.device)
        kps = self.kps[:n_frames].cpu().numpy().view(ss.KEYPOINT_DTYPE).reshape(n_frames, self.cap)
        return kps, self.desc[:n_frames].cpu().numpy(), self.counts[:n_frames].cpu().numpy()


def to_device_records(arr: np.ndarray, device) -> torch.Tensor:
    """numpy structured array -> uint8 CUDA tensor with the same bytes."""
    raw = np.ascontiguousarray(arr).view(np.uint8).reshape(len(arr), -1)
    return torch.from_numpy(raw.copy()).to(device)


def match_out(n: int, device) -> torch.Tensor:
    return torch.zeros((n, 3), dtype=torch.int32, device=device)


def match_records(t: torch.Tensor) -> np.ndarray:
    return t.cpu().numpy().astype(np.int32).view(ss.MATCH_DTYPE).reshape(-1)
