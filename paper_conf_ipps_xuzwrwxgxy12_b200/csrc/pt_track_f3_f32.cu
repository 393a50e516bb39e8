// pt_track_f3_f32.cu -- instantiations of the tracking kernel (pt_track.cuh) for 3 fibre(s)
// per voxel and f32 records; a translation unit of its own so the six (fibre count,
// precision) pairs compile in parallel.
#include "pt_track.cuh"

namespace pt {

template <>
cudaError_t launch_track_f<3, false>(const TrackArgs& a, const TrackMode& m, int num_sms, cudaStream_t st) {
    return launch_track_fh<3, false>(a, m, num_sms, st);
}

}  // namespace pt
