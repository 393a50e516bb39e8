// pt_track_f2_f16.cu -- instantiations of the tracking kernel (pt_track.cuh) for 2 fibre(s)
// per voxel and f16 records; a translation unit of its own so the six (fibre count,
// precision) pairs compile in parallel.
#include "pt_track.cuh"

namespace pt {

template <>
cudaError_t launch_track_f<2, true>(const TrackArgs& a, const TrackMode& m, int num_sms, cudaStream_t st) {
    return launch_track_fh<2, true>(a, m, num_sms, st);
}

}  // namespace pt
