"""Time the field solve (CG) at the C2 mesh size; print iterations and ms."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gen
from paper_conf_icpp_lantra0m24_b200.app import MiniFemPic
from paper_conf_icpp_lantra0m24_b200 import opp as O
mesh = gen.kuhn_duct(48, 48, 72)
sim = MiniFemPic(mesh, np.zeros((mesh["n_cells"], 3)), stream=torch.cuda.current_stream().cuda_stream)
mask, val = gen.duct_bc(mesh, wall=0.05, inlet=0.0)
t0 = time.time(); sim.field_init(mask, val); print("init s", time.time() - t0)
rng = np.random.default_rng(0)
Q = rng.uniform(200, 400, mesh["n_nodes"])
O.opp_set_dat(sim.ctx, sim.node_charge, Q, sim.nn)
for pc in (1, 0):
    for tol in (1e-6, 1e-8, 1e-10):
        sim.phase_timing(True); sim.phase_times()
        st = sim.field_solve(2e-7, tol=tol, warm_start=False, precond=bool(pc))
        ph = sim.phase_times()["field"]
        print(f"precond {pc} tol {tol:g}: it {st['iterations']} conv {st['converged']} rel {st['rel_residual']:.2e} ms {ph[0]:.3f} us/it {1e3*ph[0]/max(st['iterations'],1):.2f}")
# warm start after a perturbation of Q (a step's worth)
Q2 = Q * (1 + 0.05 * rng.standard_normal(Q.shape))
O.opp_set_dat(sim.ctx, sim.node_charge, Q2, sim.nn)
sim.phase_times()
st = sim.field_solve(2e-7, tol=1e-10, warm_start=True)
print("warm", st, sim.phase_times()["field"])
E = sim.field_host(); print("max |E|", np.abs(E).max())
for bps in (1, 2, 4, 8):
    os.environ["OPP_CG_BPS"] = str(bps)
    sim.phase_times()
    st = sim.field_solve(2e-7, tol=1e-10, warm_start=False)
    ph = sim.phase_times()["field"]
    print(f"bps {bps}: it {st['iterations']} ms {ph[0]:.3f} us/it {1e3*ph[0]/st['iterations']:.2f}")
sim.close()
sim2 = MiniFemPic(mesh, np.zeros((mesh["n_cells"], 3)), stream=torch.cuda.current_stream().cuda_stream)
sim2.field_init(mask, val)
O.opp_set_dat(sim2.ctx, sim2.node_charge, Q, sim2.nn)
sim2.phase_timing(True)
for mi in (0, 1, 50, 100, 200):
    sim2.phase_times()
    for rep in range(3):
        st = sim2.field_solve(2e-7, tol=0.0, max_iter=mi, warm_start=False)
    ph = sim2.phase_times()["field"]
    print(f"max_iter {mi}: it {st['iterations']} ms/solve {ph[0]/ph[1]:.4f}")
sim2.close()
for dbg in ("1", "2"):
    os.environ["OPP_CG_DBG"] = dbg
    sim3 = MiniFemPic(mesh, np.zeros((mesh["n_cells"], 3)), stream=torch.cuda.current_stream().cuda_stream)
    sim3.field_init(mask, val)
    sim3.phase_timing(True)
    sim3.phase_times()
    for rep in range(3):
        st = sim3.field_solve(2e-7, tol=0.0, max_iter=200, warm_start=False)
    ph = sim3.phase_times()["field"]
    print(f"dbg {dbg}: ms/solve(200 it) {ph[0]/ph[1]:.4f}")
    sim3.close()
os.environ.pop("OPP_CG_DBG")
