// rx_rebalance.cpp -- Shift Rebalancing (Sec. 5.2).
// (placeholder: filled in by the rebalancing pass commit)
#include "rx_internal.h"

namespace rx {
void rebalance_regex(RegexIR &ir) { (void)ir; }
}  // namespace rx
