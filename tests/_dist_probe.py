"""Probe script for tests/test_dist_gloo.py: started by dist.relaunch under
torchrun; every rank joins a gloo group, checks the world size and all-gathers
its rank; rank 0 prints one JSON line."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_hpca_songhcl17_b200 import dist as pdist  # noqa: E402


def main():
    n = int(sys.argv[1])
    dist.init_process_group("gloo")
    pdist.check_world(n)
    r = dist.get_rank()
    start, count = pdist.shard_range(10, n, r)
    local = torch.full((max(count, 1), 2), float(r))
    g = [torch.empty_like(local) for _ in range(n)]
    dist.all_gather(g, local)
    if r == 0:
        print(json.dumps({"world": dist.get_world_size(),
                          "ranks": [int(t[0, 0]) for t in g],
                          "env": [os.environ.get("MASTER_ADDR"), os.environ.get("LOCAL_RANK")]}))
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
