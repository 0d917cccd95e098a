"""heat-3d's resident time loop (stencil_staged.cu: heat3d_resident): the whole time loop in one
cooperative launch when every EATSS tile fits on the device at once, each tile's window kept in shared
memory across sweeps and only the face-neighbour cells reloaded after the neighbours' progress flags.

Same tiles and per-point arithmetic as the launched sweep (only space is tiled, the time loop
stays outside), so T steps in one resident launch must equal, bit for bit, T calls of one step each
(one step = two sweeps: below the resident path's threshold, so those calls launch one grid per sweep),
and both A and B must end as the fp64 oracle's (Polybench heat-3d, A and B alternate)."""
import numpy as np
import pytest
import torch

import synth
from oracle import numeric as O

pytestmark = pytest.mark.gpu
E = pytest.importorskip("paper_conf_cgo_jayaweerakwk24_b200")


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(device="cuda", dtype=torch.float32)


def host(t):
    torch.cuda.synchronize()
    return t.double().cpu().numpy()


CASES = [(120, (16, 16, 32), 0), (120, (16, 16, 32), 8), (40, (8, 8, 16), 0), (36, (4, 8, 12), 4),
         (64, (16, 16, 32), 16), (24, (8, 8, 8), 0), (52, (12, 20, 16), 32)]


@pytest.mark.parametrize("n,tiles,waf", CASES)
def test_heat3d_resident_equals_launched_sweeps(cuda_device, n, tiles, waf):
    T = 7
    A0 = synth.uniform((n, n, n), 40); B0 = synth.uniform((n, n, n), 41)
    d = E.desc_builtin("heat-3d", (n,), tsteps=T)
    d.set_exec(split_pct=50, warp_align=waf)
    assert E.launches_per_run(d, tiles) == 1  # the resident launch
    Ar, Br = dev(A0), dev(B0)
    E.run(d, tiles, [Ar, Br])
    d1 = E.desc_builtin("heat-3d", (n,), tsteps=1)
    d1.set_exec(split_pct=50, warp_align=waf)
    assert E.launches_per_run(d1, tiles) == 2  # one grid per sweep
    Al, Bl = dev(A0), dev(B0)
    for _ in range(T):
        E.run(d1, tiles, [Al, Bl])
    assert torch.equal(Ar, Al) and torch.equal(Br, Bl)
    Ao, Bo = O.heat3d(A0, B0, T)
    assert O.normwise_rel_err(host(Ar), Ao) <= 1e-5
    assert O.normwise_rel_err(host(Br), Bo) <= 1e-5


def test_heat3d_resident_linear_field_fixed_point(cuda_device):
    # a linear field is a fixed point of the 7-point Laplacian update: exact after any number of sweeps
    n = 120
    i, j, k = np.meshgrid(np.arange(n), np.arange(n), np.arange(n), indexing="ij")
    L = (3 * i - 2 * j + k).astype(np.float64)
    d = E.desc_builtin("heat-3d", (n,), tsteps=50)
    Ad, Bd = dev(L), dev(L)
    E.run(d, (16, 16, 32), [Ad, Bd])
    assert np.array_equal(host(Ad), L) and np.array_equal(host(Bd), L)


def test_heat3d_resident_repeated_runs_and_impulse(cuda_device):
    # flags are reset per run: a second run continues from the first's state exactly like one longer run
    n, tiles = 48, (16, 16, 32)
    A0 = np.zeros((n, n, n)); A0[20, 21, 22] = 1.0; B0 = A0.copy()
    d5 = E.desc_builtin("heat-3d", (n,), tsteps=5)
    Ad, Bd = dev(A0), dev(B0)
    E.run(d5, tiles, [Ad, Bd]); E.run(d5, tiles, [Ad, Bd])
    d10 = E.desc_builtin("heat-3d", (n,), tsteps=10)
    Ae, Be = dev(A0), dev(B0)
    E.run(d10, tiles, [Ae, Be])
    assert torch.equal(Ad, Ae) and torch.equal(Bd, Be)
    Ao, Bo = O.heat3d(A0, B0, 10)
    assert O.normwise_rel_err(host(Ad), Ao) <= 1e-5
