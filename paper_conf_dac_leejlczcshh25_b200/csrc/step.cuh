// step.cuh -- one incremental iteration (apply + refine) as ONE persistent
// cooperative launch: saves a launch and a kernel start per iteration on the
// latency-bound C2 path.  A rejected batch ends the kernel before the refine.
#pragma once
#include "apply.cuh"
#include "refine.cuh"

namespace igk {

union StepSmem {
  ApplySmem ap;
  RefSmem rf;
};

__global__ void __launch_bounds__(kThreads) k_step(Dev d, ApplyArgs aa, RefineArgs ra) {
  cg::grid_group grid = cg::this_grid();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  StepSmem& sm = *reinterpret_cast<StepSmem*>(smem_raw);
  if (!apply_body(d, aa, grid, sm.ap)) {
    if (blockIdx.x == 0 && threadIdx.x == 0) d.ctl->refine_skipped = 1;
    publish(d);
    return;
  }
  grid.sync();  // the refine starts from the complete applied state
  ShardArgs sh{};
  sh.mode = kModeFull;
  if (!refine_body<false>(d, ra, grid, sm.rf, sh)) publish(d);  // (the epilogue posts the notice itself)
}

}  // namespace igk
