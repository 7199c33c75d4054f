// k1_dispatch.cu -- selects the K1 implementation.
#include "kernels.hpp"

namespace paper {

cudaError_t launch_k1_direct(const StepArgs& a, bool unit_mass, cudaStream_t stream);
cudaError_t launch_k1_march(const StepArgs& a, bool unit_mass, cudaStream_t stream);
cudaError_t launch_k1_march2(const StepArgs& a, bool unit_mass, cudaStream_t stream);

cudaError_t launch_k1(K1Variant variant, const StepArgs& a, bool unit_mass, cudaStream_t stream) {
    switch (variant) {
        case K1Variant::Direct: return launch_k1_direct(a, unit_mass, stream);
        case K1Variant::March: return launch_k1_march(a, unit_mass, stream);
        case K1Variant::March2: return launch_k1_march2(a, unit_mass, stream);
    }
    return cudaErrorInvalidValue;
}

}  // namespace paper
