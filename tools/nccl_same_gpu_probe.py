# probe: can two NCCL ranks share one GPU (two processes)?
import os, sys, ctypes
sys.path.insert(0, os.getcwd())
import multiprocessing as mp
def w(rank, q, nid):
    import torch
    torch.cuda.set_device(0)
    from paper_conf_ipps_anzttdh12_b200 import bar, dist as D
    import workloads as W
    A = W.stencil7_3d(16)
    a, c = D.partition(A.n, 128, 2)[rank]
    Ar = W.stencil7_3d(16, row_lo=a, row_hi=c)
    try:
        M = D.DistMatrix(Ar, A.n, 128, 0, nid, rank, 2)
        b = torch.ones(c - a, dtype=torch.float64, device='cuda')
        x, info = M.solve(b, mode='sync-block')
        q.put((rank, 'ok', info['iters'], info['rel_res']))
    except Exception as e:
        q.put((rank, 'err', repr(e)))
if __name__ == '__main__':
    from paper_conf_ipps_anzttdh12_b200 import dist as D
    nid = D.nccl_unique_id()
    ctx = mp.get_context('spawn'); q = ctx.Queue()
    ps = [ctx.Process(target=w, args=(r, q, nid)) for r in range(2)]
    [p.start() for p in ps]
    try:
        print([q.get(timeout=120) for _ in ps])
    except Exception as e:
        print('probe timeout', e)
    [p.kill() for p in ps]
