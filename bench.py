"""bench.py -- batched ORB extract + match frames/s (and per-frame p50/p99 latency) on B200.

Contract: ``python bench.py --gpus N --steps K --warmup W`` (torchrun for
N > 1, one rank per GPU, NCCL) prints ONE JSON line on rank 0.  A step = one tick of the
configured workload: every client on this rank submits one frame, the frames are ORB-extracted
(pyramid, FAST, quadtree, orientation, blur, BRIEF) and matched -- search local points (each
client's local-map points projected into its frame, then windowed matching) or brute force --
through the C ABI.  Clients are sharded over ranks (weak scaling); with N > 1
per-frame results are gathered to rank 0 (the map owner) over NCCL on a side stream.

``--impl reference`` times the CPU oracle (oracle/, the checker) on the box's host cores on a
bounded sample of the same workload and prints the same line with "impl": "reference".
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "batched ORB extract+match frames/sec at 1/2/4/8 B200; per-frame p50 latency ms"
CONFIGS = {
    "c1": dict(shape="euroc", clients=1, nf=1000, mode="window", queries=5000, th=1.0, map=0, lf=600, lf_th=15.0,
               desc="c1: single synthetic 752x480 frame, 8 levels x1.2, 1000 ORB features, frame-to-frame matching of 600 last-frame points + search local points vs 5k local-map points (GPU projection + windowed match)"),
    "c2": dict(shape="euroc", clients=4, nf=1000, mode="window", queries=5000, th=1.0, map=0, lf=600, lf_th=15.0,
               desc="c2: EuRoC-shaped 752x480 mono stream, 4 concurrent clients per GPU, 1000 features/frame, "
                    "frame-to-frame matching of 600 last-frame points + search local points vs 5k local-map points per client "
                    "(GPU projection + windowed match)"),
    "c3": dict(shape="tum", clients=16, nf=1000, mode="window", queries=50000, th=3.0, map=0, lf=600, lf_th=15.0,
               desc="c3: TUM-RGBD-shaped 640x480, 16 clients per GPU, 1000 features, frame-to-frame matching of 600 last-frame points + search local points vs 50k local-map points (projection + windowed match)"),
    "c4": dict(shape="kitti", clients=8, stereo=True, nf=2000, mode="window", queries=10000, th=1.0, map=0,
               lf=1200, lf_th=7.0,
               desc="c4: KITTI-shaped 1241x376 stereo pairs, 8 clients per GPU, 2000 features/image, "
                    "ORB-SLAM stereo matching of every pair + frame-to-frame matching of 1200 last-frame points (stereo level gates) "
                    "+ search local points vs 10k local-map points "
                    "(left image; projection + windowed match)"),
    "c5": dict(shape="euroc", clients=8, nf=1250, mode="brute", queries=0, th=0.0, map=200000,
               desc="c5: EuRoC-shaped clients (8 per GPU, 64 over 8xB200), 1250 features, brute-force Hamming "
                    "vs a 200k shared-map descriptor set"),
}
CFG_ID = {"c1": 1, "c2": 2, "c3": 3, "c4": 4, "c5": 5}


# ----------------------------------------------------------------------------- helpers
def client_ids(rank: int, world: int, clients_per_rank: int) -> list[int]:
    """Weak scaling: rank r owns clients [r*C, (r+1)*C) (disjoint, covering all)."""
    return list(range(rank * clients_per_rank, (rank + 1) * clients_per_rank))


def pack_results(parts) -> "torch.Tensor":
    """Flatten one tick's per-frame results (uint8 views) into one send slot."""
    import torch
    return torch.cat([t.reshape(-1).view(torch.uint8) for t in parts])


def gather_to_owner(send, rank: int, world: int):
    """Per-tick result hand-off to the map-owning rank 0 (north_star: NCCL gather off the
    critical path; gloo on CPU in tests).  Returns the per-rank slots on rank 0, else None."""
    import torch
    import torch.distributed as dist
    if rank == 0:
        bufs = [torch.empty_like(send) for _ in range(world)]
        dist.gather(send, bufs, dst=0)
        return bufs
    dist.gather(send, None, dst=0)
    return None


class HostStagedGather:
    """NCCL-free per-tick result gather (``--backend gloo``): the packed send slot is copied to
    a pinned host buffer on the gather stream (gated by the tick's completion event), and a
    host thread runs the gloo gather to rank 0 once that copy has landed -- still off the
    per-frame critical path.  Lets N > 1 ranks share ONE GPU (NCCL refuses two ranks on a
    device), so the multi-rank path runs on a 1-GPU box; rank 0 keeps the last gathered slots."""

    def __init__(self, rank: int, world: int, slot_bytes: int, depth: int = 8):
        import queue

        import torch
        import torch.distributed as dist
        self.rank, self.world = rank, world
        # a process group of its own: the worker thread's gathers must never interleave with
        # the main thread's collectives (barriers, the timing all-reduce) on the default group
        self.pg = dist.new_group(backend="gloo")
        self.bufs = [torch.empty(slot_bytes, dtype=torch.uint8).pin_memory() for _ in range(depth)]
        self.recv = [[torch.empty(slot_bytes, dtype=torch.uint8) for _ in range(world)] for _ in range(depth)]
        self.events = [torch.cuda.Event() for _ in range(depth)]
        self.i = 0
        self.q = queue.Queue(maxsize=depth - 1)
        self.last = None
        self.err = None
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()

    def _run(self):
        import torch.distributed as dist
        while True:
            item = self.q.get()
            if item is None:
                return
            try:
                k = item
                self.events[k].synchronize()
                if self.rank == 0:
                    dist.gather(self.bufs[k], self.recv[k], dst=0, group=self.pg)
                    self.last = [r.clone() for r in self.recv[k]]
                else:
                    dist.gather(self.bufs[k], None, dst=0, group=self.pg)
            except Exception as e:  # pragma: no cover - surfaced by drain()
                self.err = e

    def submit(self, send, stream):
        """Enqueue the D2H copy of `send` on `stream` (already waiting for the tick)."""
        import torch
        k = self.i % len(self.bufs)
        self.i += 1
        with torch.cuda.stream(stream):
            self.bufs[k].copy_(send, non_blocking=True)
            self.events[k].record(stream)
        self.q.put(k)  # blocks when `depth - 1` gathers are outstanding (buffer reuse)

    def drain(self):
        import time as _t
        while not self.q.empty():
            _t.sleep(0.0005)
        self.q.put(None)
        self.t.join()
        if self.err:
            raise self.err


def window_inputs(p, kps, desc, counts, cfg, seed_lm, seed_lf, per_client):
    """Search-local-points and frame-to-frame inputs of one tick (synth recipes):
    a local map per client frame (left / mono images; O11 + O9) and the previous frame's
    tracked points in the same camera (O13).  kps / desc / counts: every image of the tick.
    Returns (cams [B], points, point_frame, qdesc, taken [B, cap], last_cams [B],
    lf_offsets [B+1], lf_points, lf_desc)."""
    B = kps.shape[0]
    cap = p.kp_capacity
    L = p.n_levels
    w, h = p.width, p.height
    sel = list(range(0, B, per_client))
    npl = np.array(p.n_per_level[:L])
    cm, pt, pf, qd, tk = synth.make_local_map(kps[sel], desc[sel], counts[sel], L, p.scale_factor, npl, w, h,
                                              cfg["shape"], cfg["queries"], seed=seed_lm)
    _, last, off, lp, ld = synth.make_last_frame(kps[sel], desc[sel], counts[sel], L, npl, w, h, cfg["shape"],
                                                 cfg["lf"], seed=seed_lf, cams=cm,
                                                 stereo_z=0.5 if per_client == 2 else 0.0)
    cmf = np.zeros(B, synth.CAMERA_DTYPE)
    cmf[sel] = cm
    lastf = np.zeros(B, synth.CAMERA_DTYPE)
    lastf[sel] = last
    tkf = np.zeros((B, cap), np.uint8)
    tkf[sel] = tk
    n_lf = np.zeros(B, np.int64)
    n_lf[sel] = np.diff(off)
    offf = np.concatenate([[0], np.cumsum(n_lf)]).astype(np.int32)
    return cmf, pt, (pf * per_client).astype(np.int32), qd, tkf, lastf, offf, lp, ld


def shard_range(n_map: int, rank: int, world: int) -> tuple[int, int]:
    """Map-sharded brute force (F4): rank r holds global map rows [lo, hi) (contiguous, covering)."""
    return n_map * rank // world, n_map * (rank + 1) // world


def allgather_queries(desc, counts, world: int):
    """Every rank's keypoint descriptors / counts of this tick, rank-major ([world*B, ...])."""
    import torch
    import torch.distributed as dist
    ad = torch.empty((world * desc.shape[0],) + tuple(desc.shape[1:]), dtype=desc.dtype, device=desc.device)
    ac = torch.empty((world * counts.shape[0],) + tuple(counts.shape[1:]), dtype=counts.dtype, device=counts.device)
    dist.all_gather_into_tensor(ad, desc.contiguous())
    dist.all_gather_into_tensor(ac, counts.contiguous())
    return ad, ac


def exchange_partials(top2_all, world: int):
    """top2_all [world*B, cap, 2] (this rank's shard top-2 for every rank's frames, rank-major)
    -> [world, B, cap, 2]: every shard's top-2 for THIS rank's frames (all-to-all)."""
    import torch
    import torch.distributed as dist
    recv = torch.empty_like(top2_all)
    dist.all_to_all_single(recv, top2_all.contiguous())
    return recv.reshape((world, top2_all.shape[0] // world) + tuple(top2_all.shape[1:]))


def _gen_frame(args):
    w, h, seed, stereo = args
    if stereo:
        l, r = synth.make_stereo_pair(w, h, seed)
        return np.stack([l, r])
    return synth.make_frame(w, h, seed)[None]


def make_ring_frames(cfg: dict, clients: list[int], n_slots: int, workers: int) -> np.ndarray:
    """[n_slots, images_per_step, H, W] u8, slot s = frame index s of every client."""
    w, h = synth.SHAPES[cfg["shape"]]
    stereo = bool(cfg.get("stereo"))
    jobs = [(w, h, synth.frame_seed(CFG_ID[cfg["name"]], c, s), stereo) for s in range(n_slots) for c in clients]
    if workers > 1 and len(jobs) > 8:
        import multiprocessing as mp
        with mp.get_context("fork").Pool(workers) as pool:
            imgs = pool.map(_gen_frame, jobs, chunksize=max(1, len(jobs) // (4 * workers)))
    else:
        imgs = [_gen_frame(j) for j in jobs]
    per = 2 if stereo else 1
    out = np.stack(imgs).reshape(n_slots, len(clients) * per, h, w)
    return out


class ClockSampler:
    """NVML sampling of SM clock + clock-event reasons during the timed region."""
    BAD = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown"}
    NAMES = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
             0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
             0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, device_index: int, period_s: float = 0.002):
        self.samples, self.reasons, self.ok = [], 0, False
        self.period = period_s
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover - depends on the box
            self.err = str(e)
        self._stop = threading.Event()
        self._t = None

    def _reason_bits(self):
        nv = self.nv
        fn = getattr(nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
            getattr(nv, "nvmlDeviceGetCurrentClocksThrottleReasons")
        return fn(self.h)

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                self.reasons |= int(self._reason_bits())
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self) -> dict:
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "error": getattr(self, "err", "nvml")}
        reasons = [n for b, n in self.NAMES.items() if self.reasons & b and b != 0x1]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": reasons, "samples": len(self.samples),
                "rejected": any(self.reasons & b for b in self.BAD)}


def measured_peaks() -> dict:
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return {"hbm_gbs": float(d["hbm_gbs"]), "src": "measured (MEASURED_PEAKS.json)",
                "i8_tops": 2.0 * float(d["bf16_tflops"]),
                "tc_src": "measured bf16 dense (MEASURED_PEAKS.json) x 2 (nominal int8:bf16 ratio, 4.5:2.25 POPS)"}
    except Exception:
        return {"hbm_gbs": 6650.0, "src": "fallback (B200_PROFILING.md)", "i8_tops": 4500.0,
                "tc_src": "nominal int8 dense 4.5 POPS (fallback)"}


# ----------------------------------------------------------------------------- algorithmic work
# FAST-9 work model of SURVEY.md §8(d) (N2+N3 row): >= 32 compares per detect pixel (16 ring
# pixels x 2 polarities) + the contiguity test ~= 40 integer ops per detect pixel.  (The
# kernel's own exact-score formulation issues ~52 ALU-pipe ops per pixel, the whole kernel ~95
# thread instructions per pixel with staging, NMS and output: DESIGN.md §5.)
FAST_OPS_PER_PX = 40.0
FAST_KERNEL_OPS_PER_PX = 51.5
# Hamming distance of two 256-bit descriptors: 8 POPC (XU pipe) per candidate (O9 / O13)
POPC_PER_DISTANCE = 8


def int_peaks() -> dict:
    """Measured issue rates per SM per clock (profiles/peaks_int_r02.json, scripts/micro/int_peaks.cu)."""
    path = os.path.join(ROOT, "profiles", "peaks_int_r02.json")
    try:
        with open(path) as f:
            pk = json.load(f)["peaks"]
        return {"alu": float(pk["alu_pipe_thread_ops_per_clk_per_sm"]),
                "popc": float(pk["xu_popc_thread_ops_per_clk_per_sm"]),
                "src": "measured: profiles/peaks_int_r02.json (scripts/micro/int_peaks.cu on a B200)"}
    except Exception:
        return {"alu": 64.0, "popc": 16.0, "src": "fallback: CUDA guide rates (profiles/peaks_int_r02.json missing)"}


def window_candidates(kps, counts, taken, queries, n_levels: int, max_q: int = 20000) -> tuple[int, int]:
    """(candidate distances evaluated, queries sampled) of O9 for the first max_q queries: keypoints of
    the query's frame on levels [pl-1, pl] with |x-u| < r and |y-v| < r (f32) that are not taken --
    exactly the pairs whose Hamming distance the matcher computes (8 POPC each)."""
    q = queries[:max_q]
    total = 0
    for f in np.unique(q["frame"]):
        if f < 0 or f >= kps.shape[0]:
            continue
        qq = q[q["frame"] == f]
        n = int(counts[f][-1])
        k = kps[f][:n]
        ok = taken[f][:n] == 0 if taken is not None else np.ones(n, bool)
        x, y, lev = k["x"][ok], k["y"][ok], k["level"][ok].astype(np.int32)
        for i0 in range(0, len(qq), 2048):
            b = qq[i0:i0 + 2048]
            r = b["radius"][:, None]
            dx = np.abs(np.float32(x)[None, :] - b["u"][:, None])
            dy = np.abs(np.float32(y)[None, :] - b["v"][:, None])
            gate = (lev[None, :] >= (b["pred_level"][:, None] - 1)) & (lev[None, :] <= b["pred_level"][:, None])
            total += int(((dx < r) & (dy < r) & gate).sum())
    return total, len(q)


def kernel_work(name: str, p, B: int, cand_l: list, kps_l: list, nq: int, n_map: int, nlf: int = 0) -> tuple[str, float]:
    """(bound, algorithmic bytes or work) per launch -- DESIGN.md §6 work model.
    cand_l / kps_l: candidates / kept keypoints per level summed over the batch."""
    W = [p.level_w[l] * p.level_h[l] for l in range(p.n_levels)]
    L = p.n_levels
    if name == "pyramid":  # every level l >= 1 reads level l-1 once and is written once
        return "hbm", float(B * sum(W[l - 1] + W[l] for l in range(1, L)))
    if name in ("fast", "fast_l0", "fast_l1plus"):  # ALU-bound: exact FAST-9 score of every detect pixel
        ls = {"fast": list(range(L)), "fast_l0": [0]}.get(name, list(range(1, L)))
        det = sum(B * (p.level_w[l] - 38) * (p.level_h[l] - 38) for l in ls)
        return "alu", float(det) * FAST_OPS_PER_PX
    if name == "distribute":  # read candidates, write kept keys (all levels, one launch)
        return "hbm", float(sum(4 * cand_l[l] + 4 * kps_l[l] for l in range(L)))
    if name == "describe":  # 43x43 patch per keypoint (L2 gathers) + 52 B written per keypoint
        return "hbm", float(sum(kps_l) * (43 * 43 + 4 + 52))
    if name == "match_window":  # query 20 B + descriptor 32 B read, 12 B written
        return "hbm", float(nq * 64)
    if name == "stereo":  # per left keypoint: its record + descriptor, 11x11 + 11x21 SAD pixels
        return "hbm", float(sum(kps_l)) / 2 * (20 + 32 + 121 + 231)  # half of the images are left ones
    if name == "lastframe":  # per last-frame point: 24 B point + 32 B descriptor read, 12 B written
        return "hbm", float(nlf * 68)
    if name == "lf_prepare":  # per keypoint slot: 20 B keypoint + 1 B taken read; 2 x 8 B claims, 1 B mask, 4 B index written
        return "hbm", float(B * p.kp_capacity * (20 + 1 + 16 + 1 + 4))
    if name == "lf_finish":  # per last-frame point: 12 B match + 8 B claim + 8 B angles read, 12 B written
        return "hbm", float(nlf * 40)
    if name == "project":  # map point 32 B + frame index 4 B read, query 20 B written
        return "hbm", float(nq * 56)
    if name == "match_resolve":
        return "hbm", float(nq * 12)
    if name == "brute_tc":  # s8 +-1 dot products on tcgen05: 2 x 256 ops per distance
        return "tensor", float(sum(kps_l)) * n_map * 512.0
    if name == "brute_expand":  # the tick's keypoints only (the map was prepared once): 32 B read, 256 B written
        slots = B * p.kp_capacity
        return "hbm", float(slots * (32 + 256))
    return "hbm", 0.0


# ----------------------------------------------------------------------------- our arm
def run_ours(args, cfg):
    import torch
    import torch.distributed as dist

    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline, to_device_records

    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = 0 if args.same_device else int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    backend = args.backend
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    if args.clients:
        cfg = dict(cfg, clients=args.clients)
    w, h = synth.SHAPES[cfg["shape"]]
    clients = client_ids(rank, world, cfg["clients"])
    per_client = 2 if cfg.get("stereo") else 1
    B = len(clients) * per_client  # images per step on this rank
    L = 8
    Q = cfg["queries"] * len(clients)
    window = cfg["mode"] == "window"
    pipe = OrbPipeline(w, h, cfg["nf"], L, max_frames=B * (world if args.map_shard else 1), max_queries=max(Q, 1),
                       max_map=cfg["map"], device=local)
    dist_mode = ss.SS_DIST_GRID_TOPN if args.dist == "grid" else ss.SS_DIST_QUADTREE
    pipe.set_distribution(dist_mode)
    p = pipe.params
    cap = p.kp_capacity
    props = torch.cuda.get_device_properties(dev)
    l2 = getattr(props, "L2_cache_size", 126 * 2 ** 20)
    NLF = cfg.get("lf", 0) * len(clients)  # last-frame points per tick (O13)
    MB = synth.STEREO_BASELINE.get(cfg["shape"], 0.0) if cfg.get("stereo") else 0.0
    slot_bytes = B * h * w + (Q * 68 + B * (cap + 96) + NLF * 56 + B * 100 if window else 0)
    n_slots = int(min(256, max(4, math.ceil(2 * l2 / slot_bytes))))
    if args.ring:
        n_slots = args.ring
    workers = max(1, min(32, (os.cpu_count() or 2) // max(1, world)))
    t_setup = time.time()
    frames_h = make_ring_frames(dict(cfg, name=args.config), clients, n_slots, workers)
    frames = torch.from_numpy(frames_h).to(dev)  # [R, B, H, W]
    stream = torch.cuda.Stream(dev)
    out_rows = Q if window else B * cap
    out = torch.zeros((max(out_rows, 1), 3), dtype=torch.int32, device=dev)
    cams = points = point_frame = qdesc = taken = map_desc = None
    kp_rng = np.random.default_rng(1234 + rank)
    if window:
        # "search local points" inputs per ring slot: a local map per frame (3D points,
        # projected on the GPU by ss_project_points into the WINDOW queries), descriptors, mask
        cams = torch.zeros((n_slots, B, 96), dtype=torch.uint8, device=dev)
        points = torch.zeros((n_slots, Q, 32), dtype=torch.uint8, device=dev)
        point_frame = torch.zeros((n_slots, Q), dtype=torch.int32, device=dev)
        qdesc = torch.zeros((n_slots, Q, 32), dtype=torch.uint8, device=dev)
        taken = torch.zeros((n_slots, B, cap), dtype=torch.uint8, device=dev)
        # frame-to-frame matching inputs (O13): the previous frame's tracked points per client
        lf_last = torch.zeros((n_slots, B, 96), dtype=torch.uint8, device=dev)
        lf_off = torch.zeros((n_slots, B + 1), dtype=torch.int32, device=dev)
        lf_pts = torch.zeros((n_slots, max(NLF, 1), 24), dtype=torch.uint8, device=dev)
        lf_desc = torch.zeros((n_slots, max(NLF, 1), 32), dtype=torch.uint8, device=dev)
        q_host = []
        for s in range(n_slots):
            with torch.cuda.stream(stream):
                pipe.extract(frames[s], stream=stream)
            stream.synchronize()
            kps, desc, counts = pipe.results(B)
            wi = window_inputs(p, kps, desc, counts, cfg, synth.frame_seed(CFG_ID[args.config], 1 << 16 | rank, s),
                               synth.frame_seed(CFG_ID[args.config], 2 << 16 | rank, s), per_client)
            cm_full, pt, pf, qd, tk_full, last_full, off_full, lp, ld = wi
            cams[s] = torch.from_numpy(cm_full.view(np.uint8).reshape(B, 96).copy()).to(dev)
            points[s] = torch.from_numpy(pt.view(np.uint8).reshape(Q, 32).copy()).to(dev)
            point_frame[s] = torch.from_numpy(pf).to(dev)
            qdesc[s] = torch.from_numpy(qd).to(dev)
            taken[s] = torch.from_numpy(tk_full).to(dev)
            lf_last[s] = torch.from_numpy(last_full.view(np.uint8).reshape(B, 96).copy()).to(dev)
            lf_off[s] = torch.from_numpy(off_full).to(dev)
            lf_pts[s, :NLF] = torch.from_numpy(lp.view(np.uint8).reshape(NLF, 24).copy()).to(dev)
            lf_desc[s, :NLF] = torch.from_numpy(ld).to(dev)
            if s < 16:
                q_host.append(wi)
    else:
        # shared map: rank 0 builds it from its clients' first-slot keypoints, broadcast once
        with torch.cuda.stream(stream):
            pipe.extract(frames[0], stream=stream)
        stream.synchronize()
        kps, desc, counts = pipe.results(B)
        mp = synth.make_brute_map([desc[b][: counts[b][-1]] for b in range(B)], cfg["map"], seed=77,
                                  n_from_kps=int(0.4 * cfg["map"]))
        map_desc = torch.from_numpy(mp).to(dev)
        if world > 1:
            if backend == "nccl":
                dist.broadcast(map_desc, src=0)
            else:
                mh = map_desc.cpu()
                dist.broadcast(mh, src=0)
                map_desc = mh.to(dev)
        if args.map_shard:  # F4: keep only this rank's rows (global index offset lo)
            shard_lo, shard_hi = shard_range(cfg["map"], rank, world)
            map_desc = map_desc[shard_lo:shard_hi].contiguous()
        # the shared map is server state: expanded into each context's tensor-core operand
        # layout once (ss_brute_map_prepare); every tick then expands only its keypoints
        pipe.prepare_map(map_desc, stream=stream)
        q_host = None
    torch.cuda.synchronize(dev)

    # --- one CUDA graph per ring slot (plain, timed) + an instrumented twin whose profiling
    #     events (recorded inside the graph) give every kernel's duration
    mode = ss.SS_MATCH_WINDOW if window else ss.SS_MATCH_BRUTE
    stereo = bool(cfg.get("stereo"))
    ek = ss.extract_kernels(L)
    shard = bool(args.map_shard) and not window
    eager_tail = shard and world > 1  # the sharded exchange runs eagerly after the graph (NCCL)
    mk = (["stereo_prepare", "stereo", "stereo_outliers"] if stereo else []) + \
        (["lastframe", "project"] if window else []) + \
        (["brute_expand", "brute_tc", "brute_shard_top2", "brute_parts_merge"] if shard
         else ss.match_kernels(mode, True))
    if eager_tail:
        mk = []
    BASE_M = synth.STEREO_BASELINE.get(cfg["shape"], 0.0)
    BF = float(np.float32(synth.INTRINSICS[cfg["shape"]][0] * BASE_M))
    base = ss.extract_events(L)
    kernel_ev = [(n, 1 + 2 * i, 2 + 2 * i) for i, n in enumerate(ek)] + \
                [(n, base + 2 * j, base + 2 * j + 1) for j, n in enumerate(mk)]
    n_ev = base + 2 * len(mk)
    events = [[torch.cuda.Event(enable_timing=True) for _ in range(n_ev)] for _ in range(n_slots)]
    for evs in events:  # torch creates the CUDA event lazily, at its first record
        for e in evs:
            e.record(stream)
    stream.synchronize()

    # ticks in flight: P independent contexts (scratch + outputs) on P streams, so consecutive
    # ticks overlap on the GPU the way the paper's clients share it; P = 1 serialises
    P = max(1, args.inflight)
    pipes = [pipe] + [OrbPipeline(w, h, cfg["nf"], L, max_frames=B * (world if shard else 1), max_queries=max(Q, 1),
                                  max_map=cfg["map"], device=local) for _ in range(P - 1)]
    for pp in pipes:
        pp.set_distribution(dist_mode)
        if args.match_lanes:
            ss.ss_debug_match_lanes(pp.ctx, args.match_lanes)
        if not window and pp is not pipe:
            pp.prepare_map(map_desc)
    outs = [out] + [torch.zeros_like(out) for _ in range(P - 1)]
    qbufs = [torch.zeros((max(Q, 1), 20), dtype=torch.uint8, device=dev) for _ in range(P)]  # projected queries
    lf_out = [torch.zeros((max(NLF, 1), 3), dtype=torch.int32, device=dev) for _ in range(P)]
    lf_n = [torch.zeros(B, dtype=torch.int32, device=dev) for _ in range(P)]
    lf_mask = [torch.zeros((B, cap), dtype=torch.uint8, device=dev) for _ in range(P)]
    # F4 map-sharded brute force: shard top-2 for every rank's frames, exchanged, merged
    top2_all = [torch.zeros((B * world, cap, 2), dtype=torch.int64, device=dev) for _ in range(P)] if shard else None
    bcfg = ss.brute_cfg()

    def sharded_tail(q, st):
        pp = pipes[q]
        with torch.cuda.stream(st):
            if world > 1:
                qd, qc = allgather_queries(pp.desc[:B], pp.counts[:B], world)
            else:
                qd, qc = pp.desc[:B], pp.counts[:B]
            ss.ss_match_brute_partial(pp.ctx, B * world, qd, qc, None, map_desc.shape[0], shard_lo, top2_all[q],
                                      st)  # the prepared shard
            parts = exchange_partials(top2_all[q], world) if world > 1 else top2_all[q]
            ss.ss_match_brute_merge(pp.ctx, B, pp.counts[:B], world, parts, bcfg, outs[q], st)

    npairs = B // 2 if stereo else 0
    st_out = [(torch.zeros((max(npairs, 1), cap), dtype=torch.float32, device=dev),
               torch.zeros((max(npairs, 1), cap), dtype=torch.float32, device=dev)) for _ in range(P)]
    streams = [stream] + [torch.cuda.Stream(dev) for _ in range(P - 1)]
    aux_streams = [torch.cuda.Stream(dev) for _ in range(P)]
    for q in range(1, P):  # first call outside capture (kernel attributes)
        with torch.cuda.stream(streams[q]):
            pipes[q].extract(frames[0], stream=streams[q])
    torch.cuda.synchronize(dev)

    def capture(s, prof, q=0):
        g = torch.cuda.CUDAGraph()
        pp, st, ot = pipes[q], streams[q], outs[q]
        if prof:
            ss.ss_profile_events(pp.ctx, events[s])
        # the local-map projection (cameras + map points only) runs on a forked branch beside
        # the frame-to-frame matcher (whose one CTA per frame leaves most SMs free): c2 K=20
        # 83.5k -> 86.0k frames/s, K=200 unchanged (scripts/ab_forkproj.sh); forked beside the
        # extraction instead (--fork-project 1) it cost 7 % (94.5k -> 87.4k), serial = 0
        fork = args.fork_project if window and not prof else 0
        with torch.cuda.graph(g, stream=st):
            ev0, ev1 = torch.cuda.Event(), torch.cuda.Event()
            if fork == 1:  # beside the extraction
                ev0.record(st)
                aux_streams[q].wait_event(ev0)
                pp.project(B, cams[s], points[s], point_frame[s], qbufs[q], th=cfg["th"], stream=aux_streams[q])
                ev1.record(aux_streams[q])
            pp.extract(frames[s], stream=st)
            if stereo:
                pp.stereo(frames[s], BF, BASE_M, st_out[q][0], st_out[q][1], stream=st)
            if fork == 2:  # beside the frame-to-frame matcher (one CTA per frame leaves SMs free)
                ev0.record(st)
                aux_streams[q].wait_event(ev0)
                pp.project(B, cams[s], points[s], point_frame[s], qbufs[q], th=cfg["th"], stream=aux_streams[q])
                ev1.record(aux_streams[q])
            if window:  # ORB-Matching (O13), then search local points skipping its matches (O11 + O9)
                pp.match_last_frame(B, cams[s], lf_off[s], lf_pts[s], lf_desc[s], lf_out[q], lf_n[q],
                                    last_cams=lf_last[s] if MB > 0 else None, mb=MB, th=cfg["lf_th"],
                                    min_matches=20, taken=taken[s], matched=lf_mask[q], stream=st)
                if fork:
                    st.wait_event(ev1)
                else:
                    pp.project(B, cams[s], points[s], point_frame[s], qbufs[q], th=cfg["th"], stream=st)
                pp.match_window(B, qbufs[q], qdesc[s], ot, taken=lf_mask[q], stream=st)
            elif shard:
                if not eager_tail:
                    sharded_tail(q, st)
            else:
                pp.match_brute(B, None, ot, stream=st)  # the prepared shared map
        if prof:
            assert ss.ss_profile_next(pp.ctx) == n_ev, (ss.ss_profile_next(pp.ctx), n_ev)
            ss.ss_profile_events(pp.ctx, [])
        return g

    graphs = [[capture(s, False, q) for s in range(n_slots)] for q in range(P)]
    graphs_prof = [capture(s, True, 0) for s in range(n_slots)]
    # setup, not work: upload every executable graph to the device now (cudaGraphUpload, no
    # kernel runs), so a graph's first launch inside the timed region does not pay the upload
    # (a short run replays mostly first-time (context, slot) graphs)
    import ctypes
    _rt = ctypes.CDLL("libcudart.so.12")
    for q in range(P):
        for g_ in graphs[q]:
            _rt.cudaGraphUpload(ctypes.c_void_p(g_.raw_cuda_graph_exec()), ctypes.c_void_p(streams[q].cuda_stream))
    torch.cuda.synchronize(dev)
    setup_s = time.time() - t_setup

    # --- optional gather of per-frame results to rank 0 (map owner), off the critical path
    gather_stream = torch.cuda.Stream(dev) if world > 1 else None
    if eager_tail and backend != "nccl":
        raise SystemExit("--map-shard over N > 1 ranks needs --backend nccl")

    def tick_parts(q):
        pp = pipes[q]
        return [pp.kps[:B], pp.desc[:B], pp.counts[:B], outs[q]] + ([lf_out[q], lf_n[q]] if window else [])

    staged = None
    if world > 1 and backend != "nccl":
        staged = HostStagedGather(rank, world, sum(t.numel() * t.element_size() for t in tick_parts(0)))

    def gather_step(done_ev, q):
        # side stream: waits for the tick, packs its results and gathers them to rank 0
        gather_stream.wait_event(done_ev)
        with torch.cuda.stream(gather_stream):
            send = pack_results(tick_parts(q))
            if staged is not None:
                staged.submit(send, gather_stream)
            else:
                gather_to_owner(send, rank, world)

    W_, K = args.warmup, args.steps
    ev_start = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
    ev_end = [torch.cuda.Event(enable_timing=True) for _ in range(K)]
    for e in ev_start + ev_end:  # torch creates the CUDA event lazily, at its first record
        e.record(streams[0])
    torch.cuda.synchronize(dev)

    # the timed loop launches through the runtime directly (one cudaEventRecord + cudaGraphLaunch
    # + cudaEventRecord per tick, ~4 us of host time): torch's stream context + Event.record +
    # CUDAGraph.replay cost ~28 us per tick, and in a short run the GPU waited on that enqueue
    _launch = _rt.cudaGraphLaunch
    _record = _rt.cudaEventRecord
    _launch.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
    _record.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
    raw_exec = [[ctypes.c_void_p(g_.raw_cuda_graph_exec()) for g_ in graphs[q]] for q in range(P)]
    raw_stream = [ctypes.c_void_p(streams[q].cuda_stream) for q in range(P)]

    def run_steps_raw(s0, n, marks):
        es = [ctypes.c_void_p(e.cuda_event) for e in marks[0][:n]]
        ee = [ctypes.c_void_p(e.cuda_event) for e in marks[1][:n]]
        for i in range(n):
            s = (s0 + i) % n_slots
            q = (s0 + i) % P
            st = raw_stream[q]
            if _record(es[i], st) or _launch(raw_exec[q][s], st) or _record(ee[i], st):
                raise RuntimeError("cudaGraphLaunch / cudaEventRecord failed")

    def run_steps(s0, n, marks=None):
        if marks is not None and world == 1 and not eager_tail:
            return run_steps_raw(s0, n, marks)
        for i in range(n):
            s = (s0 + i) % n_slots
            q = (s0 + i) % P
            with torch.cuda.stream(streams[q]):
                if marks is not None:
                    marks[0][i].record(streams[q])
                graphs[q][s].replay()
                if eager_tail:
                    sharded_tail(q, streams[q])
                if marks is not None:
                    marks[1][i].record(streams[q])
            if world > 1:
                ev = torch.cuda.Event()
                ev.record(streams[q])
                gather_step(ev, q)

    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(local)
    with sampler:  # started before the warm-up, so its start-up (a subprocess) leaves no idle gap before t0
        run_steps(0, W_)
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        t0.record(streams[0])
        for q in range(1, P):
            streams[q].wait_event(t0)
        t_host = time.perf_counter()
        run_steps(W_, K, (ev_start, ev_end))
        host_enqueue_ms = (time.perf_counter() - t_host) * 1e3
        for q in range(1, P):
            streams[0].wait_stream(streams[q])
        t1.record(streams[0])
        torch.cuda.synchronize(dev)
        if gather_stream is not None:
            gather_stream.synchronize()
    if staged is None and args.dump_gather:  # single rank: its own last slot
        np.save(f"{args.dump_gather}.rank{rank}.npy", pack_results(tick_parts((W_ + K - 1) % P)).cpu().numpy())
    if staged is not None:
        staged.drain()
        if args.dump_gather:  # the last tick's slots: rank 0 gathered, every rank its own
            last_q = (W_ + K - 1) % P
            own = pack_results(tick_parts(last_q)).cpu().numpy()
            np.save(f"{args.dump_gather}.rank{rank}.npy", own)
            if rank == 0:
                np.save(f"{args.dump_gather}.gathered.npy", np.stack([t_.numpy() for t_ in staged.last]))
    if world > 1:
        dist.barrier()
    T_ms = t0.elapsed_time(t1)
    step_ms = [ev_start[i].elapsed_time(ev_end[i]) for i in range(K)]
    # steady state: ticks completed between the end of step P and the end of step K (the
    # pipeline is full; excludes the ramp-up of the first P ticks in flight)
    steady = None
    if K > P + 1:
        sw = ev_end[P - 1].elapsed_time(ev_end[K - 1])
        if sw > 0:
            steady = {"value": B * world * (K - P) / (sw / 1000.0), "unit": "frames/s",
                      "window": f"end of step {P} to end of step {K} ({K - P} ticks, {P} in flight)"}
    T_max = T_ms
    if world > 1:
        tt = torch.tensor([T_ms], device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        T_max = float(tt.item())

    # --- per-kernel durations: the same K ticks replayed one at a time through the
    #     instrumented graphs (no overlap between ticks, so each kernel is timed alone)
    with torch.cuda.stream(stream):
        for i in range(K):
            graphs_prof[(W_ + i) % n_slots].replay()
    torch.cuda.synchronize(dev)
    prof_slots = sorted({(W_ + i) % n_slots for i in range(K)})
    def group(n):  # report per-level launches as level-0 / levels >= 1 / whole-pyramid totals
        if n.startswith("pyramid_l"):
            return "pyramid"
        for k in ("fast",):
            if n.startswith(k + "_l"):
                return f"{k}_l0" if n == f"{k}_l0" else f"{k}_l1plus"
        return n

    per_kernel = {}
    prof_step_ms = []
    for s in prof_slots:
        ev = events[s]
        tot = {}
        for n, a, b in kernel_ev:
            tot[group(n)] = tot.get(group(n), 0.0) + ev[a].elapsed_time(ev[b])
        for k, v in tot.items():
            per_kernel.setdefault(k, []).append(v)
        prof_step_ms.append(ev[0].elapsed_time(ev[-1]))
    avg_us = {n: 1000.0 * float(np.mean(v)) for n, v in per_kernel.items()}

    # --- work model for the roofline of the dominant kernel
    win_sample = None
    if window:  # one tick (ring slot 0) run eagerly to read back what the matcher sees
        with torch.cuda.stream(stream):
            pipe.extract(frames[0], stream=stream)
            pipe.match_last_frame(B, cams[0], lf_off[0], lf_pts[0], lf_desc[0], lf_out[0], lf_n[0],
                                  last_cams=lf_last[0] if MB > 0 else None, mb=MB, th=cfg["lf_th"], min_matches=20,
                                  taken=taken[0], matched=lf_mask[0], stream=stream)
            pipe.project(B, cams[0], points[0], point_frame[0], qbufs[0], th=cfg["th"], stream=stream)
        stream.synchronize()
        k0, _, c0 = pipe.results(B)
        qrec = qbufs[0].cpu().numpy().reshape(-1).view(ss.QUERY_DTYPE)
        win_sample = (k0, c0, lf_mask[0].cpu().numpy(), qrec)
    if getattr(args, "dump_lf_ts", None):  # instrumented builds only (scripts/lf_phases.py)
        buf = np.zeros(64 * 8 + 64 * 32 + 64 * 64, np.uint64)
        ss.lib().ss_dbg_lf_ts(buf.ctypes.data_as(ctypes.c_void_p))
        np.save(args.dump_lf_ts, buf)
    kps_h, desc_h, counts_h = pipe.results(B)  # last step's outputs
    kps_l = [int((counts_h[:, l + 1] - counts_h[:, l]).sum()) for l in range(L)]
    cand_l = [sum(len(ss.ss_debug_candidates(pipe.ctx, b, l)[0]) for b in range(B)) for l in range(L)]
    # dominant kernel = the kernel FUNCTION with the most device time per step (with
    # SS_FAST_SPLIT=1 FAST runs as two launches: level 0 beside the pyramid, levels >= 1 after
    # it); its roofline = the algorithmic work of all its launches / their summed time
    func_of = {"fast": "fast_bands", "fast_l0": "fast_bands", "fast_l1plus": "fast_bands"}
    per_func = {}
    for n_, t_ in avg_us.items():
        per_func.setdefault(func_of.get(n_, n_), []).append(n_)
    peaks = measured_peaks()
    prof_step_us = 1000.0 * float(np.mean(prof_step_ms))
    ipk = int_peaks()
    n_sm = props.multi_processor_count
    clk = sampler.summary()
    clk_mhz = float(clk.get("sm_mhz") or clk.get("sm_max_mhz") or 1965.0)
    alu_peak_tops = ipk["alu"] * n_sm * clk_mhz * 1e6 / 1e12
    popc_peak_tops = ipk["popc"] * n_sm * clk_mhz * 1e6 / 1e12

    def roof_of(func):
        members = per_func[func]
        bound = kernel_work(members[0], p, B, cand_l, kps_l, Q, cfg["map"], NLF)[0]
        work = sum(kernel_work(n_, p, B, cand_l, kps_l, Q, cfg["map"], NLF)[1] for n_ in members)
        us = sum(avg_us[n_] for n_ in members)
        name = func if len(members) == 1 else f"{func} ({' + '.join(members)})"
        share = us / prof_step_us
        if bound == "hbm":
            achieved = work / (us * 1e-6) / 1e9
            return members, {"bound": "hbm", "achieved": achieved, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                             "frac": achieved / peaks["hbm_gbs"], "traffic": None, "kernel": name,
                             "peak_src": peaks["src"], "share_of_step": share}
        if bound == "alu":
            achieved = work / (us * 1e-6) / 1e12
            return members, {"bound": "alu", "achieved": achieved, "peak": alu_peak_tops, "unit": "Tops/s",
                             "frac": achieved / alu_peak_tops, "traffic": None, "kernel": name,
                             "peak_src": f"{ipk['src']}: {ipk['alu']:.0f} ALU-pipe ops/clk/SM x {n_sm} SMs x "
                                         f"{clk_mhz:.0f} MHz (SM clock under load in this run)",
                             "work": f"{FAST_OPS_PER_PX:g} int ops per detect pixel (SURVEY.md §8(d)); the kernel's "
                                     f"score core issues ~{FAST_KERNEL_OPS_PER_PX:g} ALU-pipe ops per pixel and the "
                                     f"whole kernel ~95 thread instructions per pixel (ncu)", "share_of_step": share}
        # tensor: int8 dense peak = measured bf16 dense x 2 (the guide's nominal i8 : bf16 ratio)
        achieved = work / (us * 1e-6) / 1e12
        return members, {"bound": "tensor", "achieved": achieved, "peak": peaks["i8_tops"], "unit": "TOPS",
                         "frac": achieved / peaks["i8_tops"], "traffic": None, "kernel": name,
                         "peak_src": peaks["tc_src"],
                         "work": "512 int8 ops per keypoint x map distance (256-long +-1 dot product)",
                         "share_of_step": share}

    dom_f = max(per_func, key=lambda f_: sum(avg_us[n_] for n_ in per_func[f_]))
    members, roof = roof_of(dom_f)
    # every kernel function's roofline, largest device time first (the dominant one is `roofline`)
    rooflines = []
    for f_ in sorted(per_func, key=lambda f_: -sum(avg_us[n_] for n_ in per_func[f_])):
        r_ = roof_of(f_)[1]
        rooflines.append({k_: r_[k_] for k_ in ("kernel", "bound", "achieved", "unit", "frac", "share_of_step")})
    # integer-pipe (POPC) utilisation of the Hamming matcher (north_star): 8 POPC per candidate
    # distance it evaluates, counted exactly on a tick's inputs (a sample of its queries)
    if window and "match_window" in avg_us:
        pairs, nsamp = window_candidates(*win_sample, L)
        ops = POPC_PER_DISTANCE * pairs * (Q / max(nsamp, 1))
        ach = ops / (avg_us["match_window"] * 1e-6) / 1e12
        popc = {"kernel": "match_window", "bound": "popc (XU pipe)", "achieved": ach, "peak": popc_peak_tops,
                "unit": "Tops/s", "frac": ach / popc_peak_tops,
                "work": f"{POPC_PER_DISTANCE} POPC per candidate distance; {pairs} candidates in {nsamp} sampled "
                        f"queries of {Q} ({pairs / max(nsamp, 1):.2f} per query)",
                "peak_src": f"{ipk['src']}: {ipk['popc']:.0f} POPC/clk/SM x {n_sm} SMs x {clk_mhz:.0f} MHz"}
        for r_ in rooflines:
            if r_["kernel"] == "match_window":
                r_["popc"] = popc
    traffic_file = os.path.join(ROOT, "profiles", "dram_traffic_r02.json")
    if not os.path.exists(traffic_file):
        traffic_file = os.path.join(ROOT, "profiles", "dram_traffic_r01.json")
    if os.path.exists(traffic_file):
        try:
            with open(traffic_file) as f:
                tab = json.load(f).get(args.config, {})
            trs = [tab.get(n_) for n_ in members]
            if all(t_ is not None for t_ in trs):
                roof["traffic"] = sum(trs)  # DRAM bytes of the roofline's launches (ncu, per step)
                roof["traffic_src"] = os.path.relpath(traffic_file, ROOT)
        except Exception:
            pass

    # --- e2e through the public API with host buffers (pinned), copies inside the timed region
    # release the ring's CUDA graphs (hundreds of executable graphs make every later graph launch
    # slower, e.g. the end-to-end path's per-tick graphs)
    for row in graphs:
        for g_ in row:
            g_.reset()
    for g_ in graphs_prof:
        g_.reset()
    graphs = graphs_prof = None
    torch.cuda.synchronize(dev)
    if eager_tail:  # ss_track_tick has no cross-rank exchange: no end-to-end number for a sharded map
        e2e = {"value": None, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0,
               "note": "map-sharded brute force over N > 1 ranks needs the NCCL exchange between the partial and "
                       "merge calls; ss_track_tick serves a replicated map only"}
    else:
        # the end-to-end path keeps more ticks in flight: a tick's frames must cross PCIe before its
        # kernels start, so with only P contexts part of the GPU idles behind the copies
        Pe = max(P, args.e2e_inflight)
        e2e_pipes = [OrbPipeline(w, h, cfg["nf"], L, max_frames=B, max_queries=max(Q, 1), max_map=cfg["map"],
                                 device=local) for _ in range(Pe)]
        for pp in e2e_pipes:
            pp.set_distribution(dist_mode)
            if not window:
                pp.prepare_map(map_desc)
        e2e_streams = [torch.cuda.Stream(dev) for _ in range(Pe)]
        e2e = run_e2e(args, e2e_pipes, frames_h, q_host, map_desc, outs, B, Q, window, dev, e2e_streams,
                      th=cfg["th"], stereo=(BF, BASE_M, st_out) if stereo else None, lf=(MB, cfg.get("lf_th", 15.0)),
                      dev_map=(points, point_frame, qdesc, taken, lf_pts, lf_desc, lf_last) if window else None)
        for pp in e2e_pipes:
            pp.close()

    frames_per_step = B * world
    value = frames_per_step * K / (T_max / 1000.0)
    # kernels launched per tick: one per profiled kernel, except match_prepare, whose work O13
    # already did (ss_match_last_frame prepares the window index; its event pair is empty)
    launches_per_step = len(ek) + len(mk) - (1 if window and "lastframe" in mk else 0)
    res = {
        "metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": world, "steps": K, "warmup": W_,
        "ms_per_step": T_max / K, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "u8", "data": "synthetic",
        "config": workload_config(args, cfg, world),
        "run": {"cuda_graphs": True, "ticks_in_flight": P, "setup_s": round(setup_s, 1),
                "input_ring": {"slots": n_slots, "MiB": round(n_slots * slot_bytes / 2**20), "l2_MiB": round(l2 / 2**20)}},
        "steady_state": steady,
        "latency_ms": {"p50": float(np.percentile(step_ms, 50)), "p99": float(np.percentile(step_ms, 99)),
                       "samples": len(step_ms),
                       "note": f"per-frame latency = its tick's device time from start to end on its stream "
                               f"({P} ticks in flight; frames of a tick are processed together)",
                       "isolated_tick_ms": float(np.mean(prof_step_ms))},
        "kernels_us": avg_us,
        "kernels_note": "per-kernel device time (summed over the per-level launches; branches overlap) from "
                        "profiling events inside instrumented twin graphs replaying the same "
                        f"{K} ticks one at a time (instrumented tick {float(np.mean(prof_step_ms)):.4f} ms)",
        "roofline": roof,
        "rooflines": rooflines,
        "e2e": e2e,
        "gpu_launches": launches_per_step * K * world,
        "host_enqueue_ms": host_enqueue_ms,  # host time to enqueue the K timed ticks (graph launches + events)
        "clocks": sampler.summary(),
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        res["cpu_baseline"] = cpu_baseline(args, cfg, frames_h, q_host, budget_s=args.cpu_budget)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    for pp in pipes:
        pp.close()
    if rank == 0:
        print(json.dumps(res), flush=True)


def run_e2e(args, pipes, frames_h, q_host, map_desc, outs, B, Q, window, dev, streams, th=1.0, stereo=None,
            lf=(0.0, 15.0), dev_map=None):
    """Same ticks end to end from pinned host buffers through ONE C-ABI call per tick
    (ss_track_tick: H2D of the tick's frames and local maps, extract, stereo, projection +
    match or brute match, D2H of every output), all inside the timed region; ticks
    round-robin over the in-flight contexts/streams so copies of one tick overlap compute of
    another."""

    import torch

    from paper_conf_conext_dhakalrwcr22_b200 import ss
    P = len(pipes)
    n_host = min(len(frames_h), 8)
    cap = pipes[0].cap
    L = pipes[0].n_levels
    H, W = frames_h.shape[2], frames_h.shape[3]

    def pinned(a):
        return torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).reshape(-1).copy()).pin_memory()

    fr = [pinned(frames_h[s]) for s in range(n_host)]
    hin = [[pinned(a) for a in q_host[s % len(q_host)]] for s in range(n_host)] if window else None
    rows = Q if window else B * cap
    host_out = []
    for q in range(P):
        o = {"kps": torch.empty(B * cap * 20, dtype=torch.uint8).pin_memory(),
             "desc": torch.empty(B * cap * 32, dtype=torch.uint8).pin_memory(),
             "counts": torch.empty(B * (L + 1), dtype=torch.int32).pin_memory(),
             "matches": torch.empty(rows * 3, dtype=torch.int32).pin_memory()}
        if window:
            nlf = int(q_host[0][6][-1])
            o["lf_matches"] = torch.empty(max(nlf, 1) * 3, dtype=torch.int32).pin_memory()
            o["lf_n"] = torch.empty(B, dtype=torch.int32).pin_memory()
        if stereo:
            o["uright"] = torch.empty((B // 2) * cap, dtype=torch.float32).pin_memory()
            o["depth"] = torch.empty((B // 2) * cap, dtype=torch.float32).pin_memory()
        host_out.append(o)
    cfg = ss.window_cfg() if window else ss.brute_cfg()
    handles = [st.cuda_stream for st in streams]
    world = int(os.environ.get("WORLD_SIZE", 1))
    d2h_sep = sum(t.numel() * t.element_size() for t in host_out[0].values())
    # every output of a tick in ONE pinned block (ss_tick_io.out_packed: one D2H copy per tick
    # instead of one per output; each copy costs the DMA engine a few us whatever its size)
    n_lf = int(q_host[0][6][-1]) if window else 0
    lay = ss.ss_tick_packed_layout(pipes[0].ctx, B, Q if window else 0, n_lf, brute=not window,
                                   stereo=bool(stereo))
    packed_out = [torch.empty(int(lay[8]), dtype=torch.uint8).pin_memory() for _ in range(P)]
    # ... and the per-tick host inputs (frames, cameras, last-frame offsets) in ONE pinned block
    # per input slot (ss_tick_io.in_packed: one H2D copy per tick instead of three)
    # (frames whose width is not a multiple of 16 B, e.g. KITTI's 1241, sit in the block with
    # the row pitch rounded up to 16: the host's receive buffer layout, so the library needs no
    # unaligned copy or on-device repack)
    WP = (W + 15) // 16 * 16
    ilay = ss.ss_tick_packed_in_layout(pipes[0].ctx, B, H * WP)
    inblk = []
    for i in range(n_host):
        blk_ = torch.zeros(int(ilay[3]), dtype=torch.uint8).pin_memory()
        fview = blk_[:B * H * WP].view(B, H, WP)
        fview[:, :, :W].copy_(fr[i].view(B, H, W))
        parts = [hin[i][0], hin[i][6]] if window else []
        for j, t_ in enumerate(parts, start=1):
            blk_[int(ilay[j]):int(ilay[j]) + t_.numel()].copy_(t_)
        inblk.append(blk_)

    def measure(resident: bool, reuse: bool = False, packed: bool = True):
        """resident: the map state (local-map points, last-frame points, masks) is the server's,
        kept in HBM across ticks (dev_map, slot i); per tick only frames, camera predictions and
        the last-frame offsets come from the host."""
        ios = []
        for q in range(P):
            row = []
            o = host_out[q]
            for i in range(n_host):
                io = ss.ss_tick_io()
                io.frames, io.frame_stride, io.pitch = fr[i].data_ptr(), H * W, W
                io.reuse_graph = int(reuse)
                if stereo:
                    io.bf, io.baseline = stereo[0], stereo[1]
                if window:
                    cm, pt, pf, qd, tk, last, off, lp, ld = hin[i]
                    if resident:
                        pt, pf, qd, tk, lp, ld, last = (t_[i] for t_ in dev_map)
                    io.map_resident = int(resident)
                    io.cams, io.n_points, io.points, io.point_frame = cm.data_ptr(), Q, pt.data_ptr(), pf.data_ptr()
                    io.point_desc, io.taken, io.th = qd.data_ptr(), tk.data_ptr(), th
                    io.lf_offsets, io.lf_points, io.lf_desc = off.data_ptr(), lp.data_ptr(), ld.data_ptr()
                    io.last_cams, io.mb, io.lf_th, io.lf_min_matches = last.data_ptr(), lf[0], lf[1], 20
                    io.lf_matches, io.lf_n_matches = o["lf_matches"].data_ptr(), o["lf_n"].data_ptr()
                else:  # the map prepared on each context (ss_brute_map_prepare): io.d_map_desc = NULL
                    io.d_map_desc, io.n_map = None, map_desc.shape[0]
                io.kps, io.desc, io.counts = o["kps"].data_ptr(), o["desc"].data_ptr(), o["counts"].data_ptr()
                io.matches = o["matches"].data_ptr()
                if stereo:
                    io.uright, io.depth = o["uright"].data_ptr(), o["depth"].data_ptr()
                if packed:
                    io.out_packed = packed_out[q].data_ptr()
                    io.in_packed = inblk[i].data_ptr()
                    io.frame_stride, io.pitch = H * WP, WP
                row.append(io)
            ios.append(row)
        # bytes actually copied per tick (hin: cams, points, point_frame, qdesc, taken, last_cams,
        # lf_offsets, lf_points, lf_desc; the last cameras only in stereo, when mb > 0)
        if not window:
            h2d = fr[0].numel()
        elif resident:
            h2d = fr[0].numel() + hin[0][0].numel() + hin[0][6].numel()
        else:
            h2d = fr[0].numel() + sum(a.numel() for j, a in enumerate(hin[0]) if j != 5 or lf[0] > 0)
        if packed:  # the packed block replaces frames + cams + offsets (256-B aligned sections, 16-B row pitch)
            h2d += int(ilay[3]) - (fr[0].numel() + ((hin[0][0].numel() + hin[0][6].numel()) if window else 0))

        # the tick loop runs natively (ss_track_run: tick t = ss_track_tick on ctx t % P with
        # io slot t % n_host), so the measurement is the library's, not the Python loop's
        runner = ss.TrackRun([pp.ctx for pp in pipes], handles, B, cfg, ios)
        K = 1000  # ~60-100 ms of ticks: long enough that one host hiccup does not move the rate
        runner.run(3 * n_host if reuse else 3)  # reuse: every (ctx, slot) graph captured before timing
        torch.cuda.synchronize(dev)
        t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0.record(streams[0])
        for q in range(1, P):
            streams[q].wait_event(t0)
        h0 = time.perf_counter()
        runner.run(K)
        h1 = time.perf_counter()
        for q in range(1, P):
            streams[0].wait_stream(streams[q])
        t1.record(streams[0])
        torch.cuda.synchronize(dev)
        ms = t0.elapsed_time(t1)
        return {"value": B * world * K / (ms / 1000.0), "unit": "frames/s", "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": int(lay[8] if packed else d2h_sep), "steps": K, "ms_per_step": ms / K,
                "ticks_in_flight": P, "host_us_per_call": 1e6 * (h1 - h0) / K,
                "io": ("packed: one H2D (ss_tick_io.in_packed, frame rows at a 16-B pitch) + one D2H (out_packed) per tick"
                       if packed else "one copy per input / output")}

    path = ("ss_track_run: one ss_track_tick per tick in native code: H2D, ss_orb_extract, " +
            ("ss_stereo_match, " if stereo else "") +
            ("ss_match_last_frame, ss_project_points, ss_match_projection WINDOW" if window
             else "ss_match_projection BRUTE") + ", D2H of all outputs; no graphs")
    # raw pinned H2D bandwidth of one tick's frames, as seen by this process (diagnostic)
    _dbuf = torch.empty(fr[0].numel(), dtype=torch.uint8, device=dev)
    torch.cuda.synchronize(dev)
    _t0, _t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    _t0.record()
    for _ in range(50):
        _dbuf.copy_(fr[0], non_blocking=True)
    _t1.record()
    torch.cuda.synchronize(dev)
    h2d_gbs = fr[0].numel() * 50 / (_t0.elapsed_time(_t1) * 1e-3) / 1e9
    del _dbuf
    graph_note = ("; io.reuse_graph = 1: each (ctx, input-ring slot) tick is a cached CUDA graph replayed by "
                  "ss_track_tick (one launch per tick); direct = the same calls without graph reuse; both modes "
                  "are trial-measured, the faster one (`mode`) is measured again for `value`")
    resident = bool(window and dev_map is not None)

    def pick(res: bool):
        """Both API modes (io.reuse_graph 1 / 0) are trial-measured; the faster one is measured
        AGAIN and that fresh run is the reported value (the selection never reuses its own sample)."""
        trial_reuse, trial_direct = measure(res, True), measure(res, False)
        trial_sep = measure(res, True, packed=False)
        reuse = trial_reuse["value"] >= trial_direct["value"]
        r_ = measure(res, reuse)
        r_["mode"] = "reuse_graph" if reuse else "direct"
        r_["trials"] = {"reuse_graph": trial_reuse["value"], "direct": trial_direct["value"],
                        "reuse_graph_separate_outputs": trial_sep["value"]}
        return r_, trial_reuse, trial_direct

    if not resident:
        r, tr, td = pick(False)
        r["path"] = "pinned host -> ss_track_tick (" + path + ")" + \
            ("; the shared map is device-resident server state" if not window else "") + graph_note
        r["reuse_graph"], r["direct"] = tr, td
        r["h2d_gbs_raw"] = h2d_gbs
        return r
    r, tr, td = pick(True)
    r["path"] = ("pinned host frames + camera predictions -> ss_track_tick (" + path + "); the map state (each "
                 "client's local-map points, last-frame points, masks) is server state resident in HBM, "
                 "as the SLAM-Share server keeps the maps and clients upload only frames (P:L64, P:L68); "
                 "host_map = the same with the map state copied from the host too" + graph_note)
    r["reuse_graph"], r["direct"] = tr, td
    r["host_map"] = measure(False, True)
    r["h2d_gbs_raw"] = h2d_gbs
    return r


# ----------------------------------------------------------------------------- oracle (CPU) legs
def _oracle_job(job):
    import oracle
    (w, h, nf, frame, lm, mode, mp, th, right) = job
    p = oracle.params(w, h, nf)
    t = time.perf_counter()
    if frame is None:  # the right image of a stereo pair: handled by its left image's job
        return 0.0
    kps, desc, counts = oracle.orb_extract(p, frame)
    if right is not None:  # stereo pair: extract the right image, then O12
        kr, dr, cr = oracle.orb_extract(p, right)
        base = synth.STEREO_BASELINE["kitti"]
        bf = float(np.float32(synth.INTRINSICS["kitti"][0] * base))
        oracle.stereo_match(p, frame, right, kps, desc, counts, kr, dr, cr, bf, base)
    if mode == "window" and lm is not None:  # O13, then O11 + O9 skipping O13's matches
        cm, pt, qd, tk, last, lp, ld, mb, lf_th = lm
        off = np.array([0, len(lp)], np.int32)
        lfm, _ = oracle.match_last_frame(p, cm[None], last[None], mb, kps[None], desc[None], counts[None], tk[None],
                                         off, lp, ld, th=lf_th, min_matches=20)
        tk = tk.copy()
        tk[lfm["idx"][lfm["idx"] >= 0]] = 1
        q = oracle.project_points(p, cm[None], pt, np.zeros(len(pt), np.int32), th)
        oracle.match_window(p, kps[None], desc[None], counts[None], tk[None], q, qd)
    elif mode == "brute" and mp is not None:
        oracle.match_brute(p, desc[None], counts[None], mp, k0=0, k1=4)
    return time.perf_counter() - t


def _jobs_for(cfg, frames_h, q_host, n, w, h, mp=None):
    """Oracle jobs: one frame each (extract, then its local map projected + matched, or its
    first 4 keypoints brute-matched against the whole map)."""
    jobs = []
    S, Bimg = frames_h.shape[:2]
    per_client = 2 if cfg.get("stereo") else 1
    i = 0
    while len(jobs) < n:
        s, b = (i // Bimg) % S, i % Bimg
        lm = None
        if cfg["mode"] == "window" and q_host and b % per_client == 0:
            cm, pt, pf, qd, tk, last, off, lp, ld = q_host[s % len(q_host)]
            sel = pf == b
            mb = synth.STEREO_BASELINE.get(cfg["shape"], 0.0) if per_client == 2 else 0.0
            lm = (cm[b], pt[sel], qd[sel], tk[b], last[b], lp[off[b]:off[b + 1]], ld[off[b]:off[b + 1]], mb,
                  cfg["lf_th"])
        if per_client == 2:  # stereo: the left image's job covers the pair
            left = b % 2 == 0
            jobs.append((w, h, cfg["nf"], frames_h[s, b] if left else None, lm, cfg["mode"], mp, cfg["th"],
                         frames_h[s, b + 1] if left else None))
        else:
            jobs.append((w, h, cfg["nf"], frames_h[s, b], lm, cfg["mode"], mp, cfg["th"], None))
        i += 1
    return jobs


def cpu_baseline(args, cfg, frames_h, q_host, budget_s=15.0, mp=None):
    import multiprocessing as mpx

    import oracle
    oracle.build()
    w, h = synth.SHAPES[cfg["shape"]]
    cores = len(os.sched_getaffinity(0))
    probe = _oracle_job(_jobs_for(cfg, frames_h, q_host, 1, w, h, mp)[0])
    n = max(cores, int(budget_s * cores / max(probe, 1e-3)))
    jobs = _jobs_for(cfg, frames_h, q_host, n, w, h, mp)
    t = time.perf_counter()
    with mpx.get_context("fork").Pool(cores) as pool:
        per = pool.map(_oracle_job, jobs, chunksize=1)
    wall = time.perf_counter() - t
    return {"value": len(jobs) / wall, "unit": "frames/s", "cores": cores, "kind": "oracle",
            "sample": f"{len(jobs)} frames of the {args.config} workload (extract + " +
                      ("stereo matching of each pair + " if cfg.get("stereo") else "") +
                      (f"its {cfg.get('lf', 0)} last-frame points matched (O13), its {cfg['queries']}-point local map projected "
                       "and window-matched" if cfg["mode"] == "window"
                       else "4 keypoints brute-matched against the map") +
                      " each), one single-threaded oracle process per core",
            "median_frame_s_single_core": float(np.median(per)),
            "cpu": _cpu_model()}


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def workload_config(args, cfg, world):
    """The JSON line's `config`: the workload alone, identical on both arms (`--impl ours` and
    `--impl reference`), so the driver's ratio compares the same workload.  How an arm runs it
    (graphs, ticks in flight, the input ring's size, the oracle's sample) is in `run` /
    `cpu_baseline`."""
    window = cfg["mode"] == "window"
    per_client = 2 if cfg.get("stereo") else 1
    n_clients = cfg["clients"]  # per GPU (weak scaling)
    B = n_clients * per_client
    return {"workload": cfg["desc"], "config": args.config, "frames_per_step": B * world,
            "images_per_step_per_gpu": B, "features_per_image": cfg["nf"],
            "map_points_per_step_per_gpu": cfg["queries"] * n_clients if window else 0, "map_size": cfg["map"],
            "parallelism": f"dp{world} (clients sharded over GPUs)" +
                           (f"; result gather over {args.backend}" if world > 1 else "") +
                           ("; all ranks on one GPU (--same-device)" if args.same_device and world > 1 else ""),
            "l2": "no flush: the timed steps cycle through an input ring larger than the L2 "
                  "(sizes in run.input_ring)",
            "distribution": "grid top-N (O4g)" if args.dist == "grid" else "quadtree (O4)",
            "map": ("sharded over ranks (F4: shard top-2 for all ranks' frames, all-to-all, merge)"
                    if getattr(args, "map_shard", False) and not window else ("replicated" if not window else None))}


def run_reference(args, cfg):
    """The CPU oracle as the reference arm: each step = one bounded sample of the workload."""
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    if rank != 0:
        return
    import multiprocessing as mpx

    import oracle
    oracle.build()
    w, h = synth.SHAPES[cfg["shape"]]
    clients = client_ids(0, 1, cfg["clients"])
    frames_h = make_ring_frames(dict(cfg, name=args.config), clients, 2, max(1, os.cpu_count() or 1))
    q_host = None
    mp = None
    if cfg["mode"] == "window":
        p = oracle.params(w, h, cfg["nf"])
        q_host = []
        per_client = 2 if cfg.get("stereo") else 1
        B = frames_h.shape[1]
        for s in range(frames_h.shape[0]):
            kps, desc, counts = oracle.orb_extract_batch(p, frames_h[s])
            q_host.append(window_inputs(p, kps, desc, counts, cfg, synth.frame_seed(CFG_ID[args.config], 1 << 16, s),
                                        synth.frame_seed(CFG_ID[args.config], 2 << 16, s), per_client))
    else:
        p = oracle.params(w, h, cfg["nf"])
        kps, desc, counts = oracle.orb_extract_batch(p, frames_h[0])
        mp = synth.make_brute_map([desc[b][: counts[b][-1]] for b in range(len(desc))], cfg["map"], seed=77,
                                  n_from_kps=int(0.4 * cfg["map"]))
    cores = len(os.sched_getaffinity(0))
    B = frames_h.shape[1]
    probe = _oracle_job(_jobs_for(cfg, frames_h, q_host, 1, w, h, mp)[0])
    # frames per step: the tick's B frames, reduced so that the whole run stays within ~3 minutes
    per_step_budget = 170.0 / max(1, args.steps + args.warmup)
    n_frames = int(max(1, min(B, per_step_budget * cores / max(probe, 1e-3))))
    jobs_all = _jobs_for(cfg, frames_h, q_host, n_frames * (args.steps + args.warmup), w, h, mp)
    times = []
    with mpx.get_context("fork").Pool(min(cores, n_frames)) as pool:
        for s in range(args.warmup + args.steps):
            jobs = jobs_all[s * n_frames:(s + 1) * n_frames]
            t = time.perf_counter()
            pool.map(_oracle_job, jobs, chunksize=1)
            if s >= args.warmup:
                times.append(time.perf_counter() - t)
    T = sum(times)
    value = n_frames * len(times) / T
    res = {"impl": "reference", "metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * T / len(times),
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
           "config": workload_config(args, cfg, world),
           "cpu_baseline": {"value": value, "unit": "frames/s", "cores": min(cores, n_frames), "kind": "oracle",
                            "sample": f"{n_frames} of the tick's {B} frames per step (extract + " +
                                      (f"{cfg.get('lf', 0)} last-frame points matched + {cfg['queries']}-point "
                                       "local map projected + window-matched"
                                       if cfg["mode"] == "window" else "4 keypoints brute-matched") + " each)",
                            "cpu": _cpu_model()},
           "e2e": {"value": value, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(res), flush=True)


def main(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", choices=sorted(CONFIGS), default="c2")
    ap.add_argument("--ring", type=int, default=0, help="override the number of input ring slots")
    ap.add_argument("--inflight", type=int, default=8, help="ticks in flight (contexts/streams); 8 = the e2e depth")
    ap.add_argument("--e2e-inflight", type=int, default=8, help="ticks in flight on the end-to-end (host memory) path")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--dump-lf-ts", default=None, help=argparse.SUPPRESS)  # scripts/lf_phases.py (instrumented build)
    ap.add_argument("--map-shard", action="store_true",
                    help="brute configs: partition the map over the ranks (F4: shard top-2, all-to-all, merge)")
    ap.add_argument("--backend", choices=["nccl", "gloo"], default="nccl",
                    help="N > 1: NCCL gather on a side stream, or gloo with host-staged slots (ranks may share a GPU)")
    ap.add_argument("--same-device", action="store_true", help="every rank on cuda:0 (multi-rank test on one GPU)")
    ap.add_argument("--clients", type=int, default=0, help="override the config's clients per rank")
    ap.add_argument("--fork-project", type=int, default=2, choices=[0, 1, 2],
                    help="ring graphs: run the local-map projection on a forked branch concurrent with the "
                         "extraction (1) or with the frame-to-frame matcher (2)")
    ap.add_argument("--match-lanes", type=int, default=0, choices=[0, 1, 2, 4, 8],
                    help="lanes per WINDOW query (0 = chosen per launch)")
    ap.add_argument("--dump-gather", default="", help="write the last tick's gathered / own slots to PATH.*.npy")
    ap.add_argument("--dist", choices=["quadtree", "grid"], default="quadtree",
                    help="keypoint distribution: ORB-SLAM quadtree (O4) or grid top-N (O4g)")
    args = ap.parse_args(argv)
    assert args.warmup >= 3, "at least 3 warm-up steps"
    cfg = CONFIGS[args.config]
    if args.clients:
        cfg = dict(cfg, clients=args.clients)
    if args.impl == "reference":
        run_reference(args, cfg)
    else:
        run_ours(args, cfg)


if __name__ == "__main__":
    main()
