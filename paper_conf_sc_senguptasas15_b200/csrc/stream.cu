// stream.cu — streamed (out-of-core) mode: placeholder until the H2D shard
// streamer lands.
#include "engine.h"

namespace gr {
gr_status stream_setup(gr_graph *g, uint64_t) {
  (void)g;
  return fail(GR_EUNSUPPORTED, "streamed mode is not available in this build");
}
gr_status run_streamed(gr_graph *g, const gr_run_opts *, gr_run_stats *) {
  (void)g;
  return fail(GR_EUNSUPPORTED, "streamed mode is not available in this build");
}
void stream_destroy(gr_graph *) {}
}  // namespace gr
