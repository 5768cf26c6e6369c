// stubs.cu -- algorithms not yet implemented return GSW_EUNSUPPORTED.
#include "launch.h"

namespace gsw {

}  // namespace gsw
