// Multi-GPU slab decomposition (placeholder until the NCCL path lands).
#include <cstddef>

#include "lora_stencil.h"

extern "C" {
size_t lora_stencil_comm_id_size(void) { return 128; }
int lora_stencil_comm_get_id(void*) { return LORA_ERR_NCCL; }
int lora_stencil_comm_init(lora_comm**, int, int, const void*) { return LORA_ERR_NCCL; }
int lora_stencil_run_dist(lora_plan*, lora_comm*, const double*, double*, int64_t, void*) { return LORA_ERR_NCCL; }
void lora_stencil_comm_destroy(lora_comm*) {}
}
