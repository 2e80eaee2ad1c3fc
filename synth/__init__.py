"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NONE of the method's arithmetic (no pyramid, FAST, quadtree, BRIEF or
matching, no projection): it only draws frames, map-point queries, local-map points
(3D positions back-projected from keypoints, for O11 and O13's last-frame points) and map descriptors with the shapes
and statistics of the paper's workloads (recipe: SURVEY.md §8(d), restated in DESIGN.md §4).
"""
from .gen import (SHAPES, frame_seed, make_frame, make_frames, make_stereo_pair, make_queries,
                  make_brute_map, flip_bits, make_local_map, INTRINSICS, STEREO_BASELINE, CAMERA_DTYPE,
                  MAP_POINT_DTYPE, FRAME_POINT_DTYPE, make_last_frame, make_dotted_frame)  # noqa: F401
