// expand_w4.cu — expand kernels for 4-word path records (one TU per width keeps the
// sm_100a build parallel).
#include "expand.cuh"

namespace atf {
int launch_expand_w4(const LevelArgs& a, void* stream) { return launch_w<4>(a, stream); }
int launch_nfast_emit_w4(const LevelArgs& a, void* stream) { return launch_nfast_emit_w<4>(a, stream); }
}  // namespace atf
namespace atf {
int launch_tail_count_w4(const TailArgs& t, void* stream) { return launch_tail_count_w<4>(t, stream); }
int launch_tail_emit_w4(const TailArgs& t, void* stream) { return launch_tail_emit_w<4>(t, stream); }
}  // namespace atf
