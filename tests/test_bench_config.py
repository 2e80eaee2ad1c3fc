"""bench.py's JSON `config` names the workload only and is the same on both arms
(`--impl ours` / `--impl reference`), so the driver's ours / reference ratio compares one
workload.  CPU-only: the helper needs no device."""
import argparse
import inspect

import pytest

import bench

KEYS = {"workload", "config", "frames_per_step", "images_per_step_per_gpu", "features_per_image",
        "map_points_per_step_per_gpu", "map_size", "parallelism", "l2", "distribution", "map"}


@pytest.mark.parametrize("name", sorted(bench.CONFIGS))
@pytest.mark.parametrize("world", [1, 2])
def test_workload_config(name, world):
    a = argparse.Namespace(config=name, backend="nccl", same_device=False, dist="quadtree", map_shard=False,
                           clients=0)
    cfg = bench.CONFIGS[name]
    c = bench.workload_config(a, cfg, world)
    assert set(c) == KEYS
    per_client = 2 if cfg.get("stereo") else 1
    assert c["images_per_step_per_gpu"] == cfg["clients"] * per_client
    assert c["frames_per_step"] == world * cfg["clients"] * per_client
    assert c["config"] == name and c["workload"] == cfg["desc"]
    assert "L2" in c["l2"]


def test_both_arms_use_it():
    for fn in (bench.run_ours, bench.run_reference):
        assert '"config": workload_config(args, cfg, world)' in inspect.getsource(fn)
