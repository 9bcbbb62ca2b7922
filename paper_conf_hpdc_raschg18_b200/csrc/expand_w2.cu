// expand_w2.cu — expand kernels for 2-word path records (one TU per width keeps the
// sm_100a build parallel).
#include "expand.cuh"

namespace atf {
int launch_expand_w2(const LevelArgs& a, void* stream) { return launch_w<2>(a, stream); }
int launch_nfast_emit_w2(const LevelArgs& a, void* stream) { return launch_nfast_emit_w<2>(a, stream); }
}  // namespace atf
namespace atf {
int launch_tail_count_w2(const TailArgs& t, void* stream) { return launch_tail_count_w<2>(t, stream); }
int launch_tail_emit_w2(const TailArgs& t, void* stream) { return launch_tail_emit_w<2>(t, stream); }
}  // namespace atf
