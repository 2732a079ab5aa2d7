/*
 * split_oracle.h — the CPU oracle's own interface.  TEST INFRASTRUCTURE ONLY
 * (see split_oracle.c).  Shares nothing with include/split_ga.h.
 */
#ifndef SPLIT_ORACLE_H
#define SPLIT_ORACLE_H
#include <stdint.h>

typedef struct {
    double fitness;
    uint32_t k;          /* number of blocks m */
    int64_t var_num;     /* V = k*S2 - S1^2 = k^2 sigma^2 */
    uint64_t s1, s2;     /* sum t_j, sum t_j^2 */
    uint64_t overhead;   /* OV = sum of the cut overheads */
    uint64_t T;          /* vanilla model time */
} or_stats;

typedef struct {
    double fitness;
    uint64_t bits;
    uint32_t k;
    int64_t var_num;
} or_brute_result;

typedef struct {
    uint32_t pop_size, n_elite, tournament_size;
    double p_crossover, p_mutation;
    uint32_t k_min, k_max, front_skip, stall_generations;
    uint32_t n_islands, island_base, migration_interval, n_migrants;
} or_ga_params;

typedef struct {
    uint64_t* bits;      /* caller buffer, W words */
    double fitness;
    uint32_t k;
    int64_t var_num;
    uint64_t s1, s2, overhead;
    uint32_t generation_found, generations_run;
    uint64_t evaluations;
} or_ga_best;

void or_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
double or_dexp(double z);
int or_fitness(uint32_t n, const int64_t* lat, const int64_t* ovh, const uint64_t* bits,
               uint32_t k_min, uint32_t k_max, or_stats* out);
double or_fitness_value(uint32_t n, const int64_t* lat, const int64_t* ovh, const uint64_t* bits,
                        uint32_t k_min, uint32_t k_max);
void or_fitness_batch(uint32_t n, const int64_t* lat, const int64_t* ovh, const uint64_t* bits,
                      uint64_t n_cand, uint32_t k_min, uint32_t k_max, double* f_out);
double or_fitness_from(uint32_t k, int64_t V, int64_t OV, int64_t T);
int or_brute(uint32_t n, const int64_t* lat, const int64_t* ovh, uint32_t k_min, uint32_t k_max,
             or_brute_result* res, int64_t* minV_per_k, uint64_t* argminV_per_k);
int or_dp(uint32_t n, const int64_t* lat, int64_t delta, uint32_t k_max, int64_t* Vstar);
uint64_t or_count_fixed_k(uint32_t n, uint32_t k);
void or_heatmap2(uint32_t n, const int64_t* lat, const int64_t* ovh, int64_t* var_out, uint64_t* ov_out,
                 double* fit_out);
int or_ga_migrate(uint32_t W, uint32_t N, uint32_t I, uint32_t K, uint32_t island_base,
                  uint64_t* pop, double* fit);
int or_ga_run(uint32_t n, const int64_t* lat, const int64_t* ovh, const or_ga_params* p,
              uint32_t generations, uint64_t seed, or_ga_best* best,
              uint64_t* final_pop, double* final_fit);
#endif
