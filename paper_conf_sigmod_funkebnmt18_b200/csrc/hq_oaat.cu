// hq_oaat.cu -- operator-at-a-time execution of an hq_plan (placeholder).
#include "hq_internal.h"
void hq_run_oaat(hq_ctx*, const hq_plan*, hq_result*) {
  HQ_THROW(HQ_ERR_UNSUPPORTED, "operator-at-a-time execution not built yet");
}
