"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NONE of the method's arithmetic (no pyramid, FAST, quadtree, BRIEF or
matching): it only draws frames, map-point queries and map descriptors with the shapes
and statistics of the paper's workloads (recipe: SURVEY.md §8(d), restated in DESIGN.md §4).
"""
from .gen import (SHAPES, frame_seed, make_frame, make_frames, make_stereo_pair, make_queries,
                  make_brute_map, flip_bits)  # noqa: F401
