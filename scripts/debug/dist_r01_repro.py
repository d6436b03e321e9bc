"""Reproduce round 1's open item: the round-1 DistributedEngine (scripts/debug/dist_r01.py,
verbatim from commit 8c59b2c) with its root build-fault checks moved after the fetch,
two ranks (gloo) on one GPU, the multi-pipeline TPC-H queries at SF 1.  Prints every
late fault with the build that raised it."""
import os
import socket
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import torch.multiprocessing as mp  # noqa: E402

QS = ["tpch_q4", "tpch_q13", "tpch_q17", "tpch_q18", "tpch_q19", "tpch_q21"]


def worker(rank, world, port, q, reps):
    import torch
    import torch.distributed as dist

    import hqgen
    import dist_r01
    from paper_conf_sigmod_funkebnmt18_b200 import hq
    from paper_conf_sigmod_funkebnmt18_b200.engine import fetch
    from paper_conf_sigmod_funkebnmt18_b200.queries import QUERIES, load_tables

    trace = os.environ.get("HQ_REPRO_TRACE") == "1"
    log_t = torch.zeros((256, 32), dtype=torch.int64, device="cuda") if trace else None
    labels = []

    def probe(E, what):
        """Enqueue (no sync) a read of every root build's fault words at this stream point."""
        if not trace or E.rank != 0 or len(labels) >= 256:
            return
        hs = list(E._built) + [h for h in E._extra]
        E.ctx.gather_faults(hs, [], log_t[len(labels)].data_ptr())
        labels.append((what, len(hs)))

    if os.environ.get("HQ_REPRO_CLONE") == "1":
        # experiment: the root broadcasts torch-owned copies of its slot arrays instead of
        # the library-owned arrays themselves (gloo then never writes the root's tables)
        orig_bcast = dist_r01.dist.broadcast

        def bcast_clone(t, src=0, **kw):
            if dist.get_rank() == src and t.dtype == torch.uint8:
                c = t.clone()
                return orig_bcast(c, src=src, **kw)
            return orig_bcast(t, src=src, **kw)
        dist_r01.dist.broadcast = bcast_clone

    class Late(dist_r01.DistributedEngine):
        def __init__(self, *a, **k):
            super().__init__(*a, **k)
            self._extra = []

        def hash(self, *a, **k):
            h = super().hash(*a, **k)
            probe(self, "hash")
            return h

        def hashes(self, *a, **k):
            hs = super().hashes(*a, **k)
            probe(self, "hashes")
            return hs

        def hash_from(self, *a, **k):
            h = super().hash_from(*a, **k)
            probe(self, "hash_from")
            return h

        def run(self, *a, **k):
            r = super().run(*a, **k)
            probe(self, "run")
            return r

        def gather(self, *a, **k):
            r = super().gather(*a, **k)
            probe(self, "gather")
            return r

        def finish(self, res, pb):
            built = list(self._built)
            self._built.clear()
            self._extra = built
            probe(self, "finish:start")
            out = super().finish(res, pb)  # the round-1 finish with an empty check list
            probe(self, "finish:after-fetch")
            faults = []
            for i, h in enumerate(built):
                try:
                    h.info()
                except hq.HQError as e:
                    faults.append((i, h.meta().nkeys, h.meta().capacity, h.meta().layout, str(e)))
            return out, faults

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ctx = hq.Context(0)
    log = []
    for rep in range(reps):
        for qn in QS:
            qq = QUERIES[qn]
            n = hqgen.table_rows(qq.fact, 1.0)
            rng = dist_r01.partition(n, rank, world)
            tables = load_tables(ctx, qq, 1.0, fact_range=rng, skip_dims=rank != 0)
            E = Late(ctx, tables)
            try:
                res, pb = qq.run(E)
                out, faults = E.finish(res, pb)
            except Exception as e:  # noqa: BLE001
                faults = [("exception", repr(e)[:300])]
            if faults:
                log.append((rep, qn, faults))
            if trace and rank == 0 and faults:
                torch.cuda.synchronize()
                lt = log_t.cpu().tolist()
                for i, (what, nh) in enumerate(labels):
                    bits = [k for k in range(16) if lt[i][k]]
                    log.append(("trace", qn, i, what, nh, bits))
            labels.clear()
            if trace:
                log_t.zero_()
    q.put((rank, log))
    dist.barrier()
    dist.destroy_process_group()


def main():
    reps = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=worker, args=(r, 2, port, q, reps)) for r in range(2)]
    for p in ps:
        p.start()
    for _ in ps:
        rank, log = q.get(timeout=1800)
        print("rank", rank, "late faults:", len(log))
        for e in log:
            print("  ", e)
    for p in ps:
        p.join()


if __name__ == "__main__":
    main()
