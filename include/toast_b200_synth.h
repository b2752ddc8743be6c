/*
 * toast_b200_synth.h — on-device generator of the seeded synthetic timestream used by bench.py
 * and the tests (SURVEY.md 8(d) input recipe).  NOT part of the method's ABI: it computes none
 * of the pointing->map arithmetic; it exists so the 52 GB C4 timestream need not cross PCIe.
 *
 *   out[d][s] = sigma[d] * ((h >> 11) * 2^-52 - 1),
 *   h = mix(mix(mix(seed + G (stream_id + 1)) + G (det_ids[d] + 1)) + G (s + 1)),
 * mix = the SplitMix64 finaliser, G = 0x9E3779B97F4A7C15, all arithmetic mod 2^64 — the same
 * counter hash as paper_conf_sc_demeurekktbb23_b200/synth.py (bit-identical; the TOD stream of
 * the recipe is stream_id = 1).
 *   out      [n_det][n_samp] f64, device, written
 *   sigma    [n_det] f64, device;  det_ids [n_det] i64, device (global detector ids)
 * Asynchronous on `stream`.  Returns 0, -1 (bad argument, nothing launched) or -2 (launch error).
 */
#ifndef TOAST_B200_SYNTH_H
#define TOAST_B200_SYNTH_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

int toast_synth_tod(double *out, const double *sigma, const int64_t *det_ids, int64_t n_det, int64_t n_samp,
                    uint64_t seed, uint64_t stream_id, void *stream);

#ifdef __cplusplus
}
#endif

#endif /* TOAST_B200_SYNTH_H */
