// pt_track_f3.cu -- instantiations of the tracking kernel (pt_track.cuh) for 3 fibre(s) per
// voxel, fp32 and fp16 records; a translation unit of its own so the fibre counts compile in
// parallel.
#include "pt_track.cuh"

namespace pt {

template <>
cudaError_t launch_track_f<3>(const TrackArgs& a, const TrackMode& m, bool half, int num_sms, cudaStream_t st) {
    return half ? launch_track_fh<3, true>(a, m, num_sms, st) : launch_track_fh<3, false>(a, m, num_sms, st);
}

}  // namespace pt
