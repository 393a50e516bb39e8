// pt_track_f1_f16.cu -- instantiations of the tracking kernel (pt_track.cuh) for 1 fibre(s)
// per voxel and f16 records; a translation unit of its own so the six (fibre count,
// precision) pairs compile in parallel.
#include "pt_track.cuh"

namespace pt {

template <>
cudaError_t launch_track_f<1, true>(const TrackArgs& a, const TrackMode& m, int num_sms, cudaStream_t st) {
    return launch_track_fh<1, true>(a, m, num_sms, st);
}

}  // namespace pt
