"""Worker of tests/test_gpu_next.py::test_two_rank_sharded_engine_on_one_gpu
(one process per rank; torch.multiprocessing.spawn needs an importable
function)."""
import json
import os


def sharded_rank(rank, world, port, outdir):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_ayresc18_b200.parallel import ShardedTreeLikelihood
    from workloads import make_workload
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        torch.cuda.set_stream(torch.cuda.Stream())      # distinct streams per rank
        w = make_workload(tree_kind="random", n=100, p=9_001, model="gtr", c=4, seed=23)
        sh = ShardedTreeLikelihood(w.n, w.p, w.s, w.c, rank, world, precision=64, deterministic_reduce=True)
        sh.set_model_params(w.model, w.rates, w.cat_weights)
        sh.set_tips(w.tips)
        sh.set_pattern_weights(w.pattern_weights)
        sh.set_tree(w.tree.parent, w.tree.blen)
        lnl = sh.loglik()
        sh.close()
        with open(os.path.join(outdir, f"rank{rank}.json"), "w") as f:
            json.dump({"lnl": lnl, "slice": [sh.lo, sh.hi]}, f)
    finally:
        dist.destroy_process_group()
