// Small-tile AC-ESC (reading R32): the AC-ESC kernel of esc.cu compiled a second time
// with 128 threads x 4 sorted elements (CAP = 512, the paper's "256/512 non-zeros" block
// with one product each) for the blocks of at most 512 products.  Such a block is one
// local ESC iteration (Alg. 2 draws everything at once, L206), and the 2,048-slot tile
// of the default build would sort three quarters padding.  Everything lives in its own
// namespace, so the two instantiations of the block-level primitives never mix.
// The tile is fixed by the block's product count, which the decomposition fixes:
// results stay bit-stable and identical for every GPU count.
#define ACS_ITEMS 4
#define ACS_KEEP_PER_THREAD 1
#define ESC_MIN_BLOCKS 8
#define acs acs_small
#include "esc.cu"
#undef acs

static_assert(acs_small::CAP == acs_small::CAP_SMALL, "small tile");

// entry point for plan.cu (acs::EscArgs and acs_small::EscArgs are the same struct): the
// persistent grid walks the small list (esc_list_small / esc_count_small / esc_next_small)
void acs_launch_esc_small(const void* args, bool f64, cudaStream_t st) {
  acs_small::EscArgs a = *static_cast<const acs_small::EscArgs*>(args);
  if (!a.hash_done || !a.esc_list_small) return;
  a.esc_list = a.esc_list_small;
  a.esc_count = a.esc_count_small;
  a.esc_next = a.esc_next_small;
  acs_small::launch_esc(a, f64, st);
}
