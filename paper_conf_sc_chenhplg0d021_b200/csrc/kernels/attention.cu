// On-the-fly attention (placeholder until the tcgen05 kernel lands).
#include "../internal.h"
namespace et {
int attn_short_max(int d_k) { return d_k == 64 ? 256 : 128; }
et_status attention_run(const AttnArgs&, cudaStream_t) { return fail(ET_ERR_UNSUPPORTED, "attention: not built yet"); }
}  // namespace et
