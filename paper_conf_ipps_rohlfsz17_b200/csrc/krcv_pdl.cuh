// krcv_pdl.cuh -- programmatic dependent launch (PDL) for the pipeline's
// kernel chain.  The host launches each dependent kernel with
// cudaLaunchAttributeProgrammaticStreamSerialization (launch_pdl in
// krcv_device.cu), so its launch and CTA scheduling overlap the tail of the
// kernel before it (also inside a captured CUDA graph); the kernel itself
// calls pdl_wait() before touching any global memory, which blocks until the
// preceding grid has completed and its writes are visible -- the same
// ordering as a plain stream, minus the launch gap.  Without the attribute
// pdl_wait() returns at once.
#pragma once

namespace krcv {

__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

}  // namespace krcv
