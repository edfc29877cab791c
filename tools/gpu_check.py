"""GPU diagnosis: run each model isolated on the GPU and compare every node with the
oracle (uses oracle/: test tooling, not product)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_sosp_ngd023_b200 import _lib as L
from workload import archs, rng
from oracle import infer

names = sys.argv[1:] or ["toy", "resnet18", "mobilenet_v2", "squeezenet1_1", "resnet50", "densenet121", "inception_v3"]
e = L.Engine(num_clients=1)
DTS = [int(x) for x in os.environ.get("DTS", "0").split(",")]
for name in names:
    for dt in DTS:
        g = archs.build(name); P = rng.model_params(g)
        t0 = time.time()
        mid = e.register_model(g, P, dtype=dt, name=f"{name}-{dt}")
        x = rng.image(g, 0)
        out, kt = e.run_isolated(mid, x, timing=True)
        ref_all = infer.forward(g, P, x, dtype="bf16" if dt == 0 else "fp32", return_all=True)
        ref = ref_all[g.output].reshape(-1)
        err = np.abs(out - ref); tol = (2e-2 + 1e-2 * np.abs(ref)) if dt == 0 else (1e-4 + 1e-4 * np.abs(ref))
        ks = e.kernels(mid)
        order = np.argsort(-kt)[:8]
        print("   top kernels:", ", ".join(f"{ks[i]['name']}#{i} g{ks[i]['grid']} {kt[i]/1e3:.1f}us" for i in order))
        out2, kt = e.run_isolated(mid, x, timing=True)
        print("   by kind:", {k: round(sum(kt[i] for i in range(len(ks)) if ks[i]['name'] == k)/1e3, 1) for k in set(x['name'] for x in ks)})
        print(f"{name} dt={dt} reg {time.time()-t0:.1f}s kernels={len(kt)} sum_t={kt.sum()/1e3:.1f}us maxerr={err.max():.3e} "
              f"ok={np.all(err <= tol)} refstd={ref.std():.3f}", flush=True)
        if not np.all(err <= tol):
            for n in g.nodes[:-1]:
                if n['op'] == 'concat': continue
                got = e.debug_node(mid, n['id'], n['out'])
                r = ref_all[n['id']]
                d = np.abs(got - r).max()
                print(f"   node {n['id']:3d} {n['op']:8s} {n['name']:40s} maxerr {d:.3e} refmax {np.abs(r).max():.3e}")
                if d > 0.1 * max(1, np.abs(r).max()): break
e.shutdown()
