/*
 * datagen/tpchgen.c -- seeded, counter-based synthetic TPC-H columns (shared input
 * infrastructure, no method arithmetic).  Recipe: SURVEY.md 8(c).2 "TPC-H"; the
 * paper runs TPC-H; BASELINE config 4 uses Q1/Q3/Q5/Q6.
 *
 * Deviations from dbgen (result-neutral for parity, reading O2): dense
 * orderkeys with exactly 4 lines per order, uniform FKs.  Decimals are scale-2
 * int64 (reading O5): l_quantity = 100*(1..50), l_discount 0..10, l_tax 0..8,
 * prices in cents.  Dates are int32 yyyymmdd.
 */
#include <stdint.h>
#include <math.h>

uint64_t ddqgen_hash(uint64_t seed, uint32_t table, uint32_t draw, uint64_t i);
int32_t ddqgen_datekey_of_index(int64_t idx);
int ddqgen_dict_size(int dict);
int64_t ddqgen_key_of(int key_mode, int64_t n, int64_t i); /* ssbgen.c: dense / sparse keys */
int ddqgen_type_code(int s1, int s2, int s3);               /* ssbgen.c: p_type dictionary */

enum { TH_NATION = 11, TH_REGION = 12, TH_CUSTOMER = 13, TH_SUPPLIER = 14, TH_PART = 15,
       TH_ORDERS = 16, TH_LINEITEM = 17, TH_CALENDAR = 18, TH_PARTSUPP = 19 };
/* TH_PARTSUPP (TPC-H Q2): 4 rows per part; row j = (part j / 4, the (j % 4)-th supplier
 * of the TPC-H rule ps_suppkey = (ps_partkey + i * (S/4 + (ps_partkey - 1) / S)) % S + 1
 * on dense keys), ps_supplycost uniform 1.00 .. 1000.00 (scale 2). */
enum { PS_PARTKEY = 0, PS_SUPPKEY, PS_SUPPLYCOST };
/* TH_CALENDAR: the date dimension of TPC-H's date domain (one row per day
 * 1992-01-01 .. 1998-12-31, as SSB's date table): d_datekey yyyymmdd, d_year.
 * Q7's extract(year from l_shipdate) joins it (reading O34). */
enum { CAL_DATEKEY = 0, CAL_YEAR };
#define N_CALENDAR 2557
enum { N_NATIONKEY = 0, N_NAME, N_REGIONKEY };
enum { R_REGIONKEY = 0, R_NAME };
enum { HC_CUSTKEY = 0, HC_NATIONKEY, HC_MKTSEGMENT };
enum { HS_SUPPKEY = 0, HS_NATIONKEY, HS_ACCTBAL };            /* s_acctbal -999.99 .. 9999.99 */
enum { HP_PARTKEY = 0, HP_RETAILPRICE, HP_MFGR, HP_TYPE, HP_SIZE }; /* TPC-H part attributes */
enum { O_ORDERKEY = 0, O_CUSTKEY, O_ORDERDATE, O_SHIPPRIORITY, O_ORDERPRIORITY };
enum { L_ORDERKEY = 0, L_PARTKEY, L_SUPPKEY, L_LINENUMBER, L_QUANTITY, L_EXTENDEDPRICE,
       L_DISCOUNT, L_TAX, L_RETURNFLAG, L_LINESTATUS, L_SHIPDATE, L_COMMITDATE, L_RECEIPTDATE,
       L_NCOLS };
enum { DRH_NATION = 1, DRH_SEGMENT = 2, DRH_CUST = 10, DRH_ODATE = 11, DRH_PART = 12, DRH_SUPP = 13,
       DRH_QTY = 14, DRH_DISC = 15, DRH_TAX = 16, DRH_SHIP = 17, DRH_RECEIPT = 18, DRH_COMMIT = 19,
       DRH_RFLAG = 20, DRH_OPRIO = 21, DRH_MFGR = 22, DRH_TYPE = 23, DRH_SIZE = 24, DRH_ACCTBAL = 25,
       DRH_PSCOST = 26 };

#define N_ORDERDATES 2406
#define CUTOFF_19950617 19950617

/* sorted nation dictionary code of each nationkey (DICT_NATION is bytewise sorted) */
static const int NATION_CODE[25] = {
  /* ALGERIA ARGENTINA BRAZIL CANADA EGYPT ETHIOPIA FRANCE GERMANY INDIA INDONESIA IRAN IRAQ
     JAPAN JORDAN KENYA MOROCCO MOZAMBIQUE PERU CHINA ROMANIA SAUDI ARABIA VIETNAM RUSSIA
     UNITED KINGDOM UNITED STATES */
  0, 1, 2, 3, 5, 6, 7, 8, 9, 10, 11, 12, 13, 14, 15, 16, 17, 18, 4, 19, 21, 24, 20, 22, 23};
static const int NATION_REGION_H[25] = {0, 1, 1, 1, 4, 0, 3, 3, 2, 2, 4, 4, 2, 4, 0,
                                        0, 0, 1, 2, 3, 4, 2, 3, 3, 1};

static int64_t scaled_h(double sf, double base) {
  double v = floor(base * sf + 0.5); return v < 1 ? 1 : (int64_t)v;
}
int64_t ddqgen_tpch_rows(int table, double sf) {
  switch (table) {
    case TH_NATION: return 25;
    case TH_REGION: return 5;
    case TH_CUSTOMER: return scaled_h(sf, 150000.0);
    case TH_SUPPLIER: return scaled_h(sf, 10000.0);
    case TH_PART: return scaled_h(sf, 200000.0);
    case TH_ORDERS: return scaled_h(sf, 1500000.0);
    case TH_LINEITEM: return 4 * scaled_h(sf, 1500000.0);
    case TH_CALENDAR: return N_CALENDAR;
    case TH_PARTSUPP: return 4 * scaled_h(sf, 200000.0);
  }
  return -1;
}
int ddqgen_tpch_width(int table, int col) {
  switch (table) {
    case TH_NATION: return (col >= 0 && col <= N_REGIONKEY) ? 4 : 0;
    case TH_REGION: return (col >= 0 && col <= R_NAME) ? 4 : 0;
    case TH_CUSTOMER: return (col >= 0 && col <= HC_MKTSEGMENT) ? 4 : 0;
    case TH_SUPPLIER: return col == HS_ACCTBAL ? 8 : (col >= 0 && col <= HS_NATIONKEY) ? 4 : 0;
    case TH_PART: return col == HP_RETAILPRICE ? 8 : (col >= 0 && col <= HP_SIZE) ? 4 : 0;
    case TH_PARTSUPP: return col == PS_SUPPLYCOST ? 8 : (col == PS_PARTKEY || col == PS_SUPPKEY) ? 4 : 0;
    case TH_ORDERS: return (col >= 0 && col <= O_ORDERPRIORITY) ? 4 : 0;
    case TH_LINEITEM:
      if (col < 0 || col >= L_NCOLS) return 0;
      return (col >= L_QUANTITY && col <= L_TAX) ? 8 : 4;
    case TH_CALENDAR: return (col == CAL_DATEKEY || col == CAL_YEAR) ? 4 : 0;
  }
  return 0;
}
static inline int64_t retailprice_h(int64_t k) {
  return 90000 + ((k / 10) % 20001) + 100 * (k % 1000);
}

static void gen_rows_h(uint64_t seed, double sf, int table, int col, int64_t b, int64_t e, void* out, int km) {
  int32_t* o32 = (int32_t*)out; int64_t* o64 = (int64_t*)out; int64_t i;
  int64_t n_c = ddqgen_tpch_rows(TH_CUSTOMER, sf), n_s = ddqgen_tpch_rows(TH_SUPPLIER, sf);
  int64_t n_p = ddqgen_tpch_rows(TH_PART, sf), n_o = ddqgen_tpch_rows(TH_ORDERS, sf);
  for (i = b; i < e; i++) {
    int64_t k = i - b;
    switch (table) {
      case TH_NATION:
        o32[k] = col == N_NATIONKEY ? (int32_t)i : col == N_NAME ? NATION_CODE[i] : NATION_REGION_H[i];
        break;
      case TH_REGION: o32[k] = (int32_t)i; break; /* region dict sorted == regionkey order */
      case TH_CALENDAR: {
        const int32_t dk = ddqgen_datekey_of_index(i);
        o32[k] = col == CAL_DATEKEY ? dk : dk / 10000;
      } break;
      case TH_CUSTOMER:
        if (col == HC_CUSTKEY) o32[k] = (int32_t)ddqgen_key_of(km, n_c, i);
        else if (col == HC_NATIONKEY) o32[k] = (int32_t)(ddqgen_hash(seed, table, DRH_NATION, (uint64_t)i) % 25u);
        else o32[k] = (int32_t)(ddqgen_hash(seed, table, DRH_SEGMENT, (uint64_t)i) % 5u);
        break;
      case TH_SUPPLIER:
        if (col == HS_SUPPKEY) o32[k] = (int32_t)ddqgen_key_of(km, n_s, i);
        else if (col == HS_ACCTBAL) o64[k] = -99999 + (int64_t)(ddqgen_hash(seed, table, DRH_ACCTBAL, (uint64_t)i) % 1099999u);
        else o32[k] = (int32_t)(ddqgen_hash(seed, table, DRH_NATION, (uint64_t)i) % 25u);
        break;
      case TH_PART:
        if (col == HP_PARTKEY) o32[k] = (int32_t)ddqgen_key_of(km, n_p, i);
        else if (col == HP_RETAILPRICE) o64[k] = retailprice_h(i + 1);
        else if (col == HP_MFGR) o32[k] = (int32_t)(ddqgen_hash(seed, table, DRH_MFGR, (uint64_t)i) % 5u); /* sorted */
        else if (col == HP_SIZE) o32[k] = 1 + (int32_t)(ddqgen_hash(seed, table, DRH_SIZE, (uint64_t)i) % 50u);
        else {
          const uint64_t h = ddqgen_hash(seed, table, DRH_TYPE, (uint64_t)i) % 150u;
          o32[k] = ddqgen_type_code((int)(h / 25), (int)(h / 5 % 5), (int)(h % 5));
        }
        break;
      case TH_PARTSUPP: {
        const int64_t p = i / 4, pk = p + 1, j = i % 4;
        const int64_t sd = (pk + j * (n_s / 4 + (pk - 1) / n_s)) % n_s; /* 0-based supplier index */
        if (col == PS_PARTKEY) o32[k] = (int32_t)ddqgen_key_of(km, n_p, p);
        else if (col == PS_SUPPKEY) o32[k] = (int32_t)ddqgen_key_of(km, n_s, sd);
        else o64[k] = 100 + (int64_t)(ddqgen_hash(seed, table, DRH_PSCOST, (uint64_t)i) % 99901u);
      } break;
      case TH_ORDERS:
        if (col == O_ORDERKEY) o32[k] = (int32_t)ddqgen_key_of(km, n_o, i);
        else if (col == O_CUSTKEY)
          o32[k] = (int32_t)ddqgen_key_of(km, n_c, (int64_t)(ddqgen_hash(seed, TH_ORDERS, DRH_CUST, (uint64_t)i) % (uint64_t)n_c));
        else if (col == O_ORDERDATE)
          o32[k] = ddqgen_datekey_of_index((int64_t)(ddqgen_hash(seed, TH_ORDERS, DRH_ODATE, (uint64_t)i) % N_ORDERDATES));
        else if (col == O_ORDERPRIORITY) /* dict "1-URGENT".."5-LOW" (sorted == priority) */
          o32[k] = (int32_t)(ddqgen_hash(seed, TH_ORDERS, DRH_OPRIO, (uint64_t)i) % 5u);
        else o32[k] = 0;
        break;
      case TH_LINEITEM: {
        int64_t o = i / 4;
        int64_t od = (int64_t)(ddqgen_hash(seed, TH_ORDERS, DRH_ODATE, (uint64_t)o) % N_ORDERDATES);
        int64_t ship = od + 1 + (int64_t)(ddqgen_hash(seed, TH_LINEITEM, DRH_SHIP, (uint64_t)i) % 121u);
        int64_t rcpt = ship + 1 + (int64_t)(ddqgen_hash(seed, TH_LINEITEM, DRH_RECEIPT, (uint64_t)i) % 30u);
        int64_t pk = 1 + (int64_t)(ddqgen_hash(seed, TH_LINEITEM, DRH_PART, (uint64_t)i) % (uint64_t)n_p);
        int64_t qty = 100 * (1 + (int64_t)(ddqgen_hash(seed, TH_LINEITEM, DRH_QTY, (uint64_t)i) % 50u));
        switch (col) {
          case L_ORDERKEY: o32[k] = (int32_t)ddqgen_key_of(km, n_o, o); break;
          case L_PARTKEY: o32[k] = (int32_t)ddqgen_key_of(km, n_p, pk - 1); break;
          case L_SUPPKEY:
            o32[k] = (int32_t)ddqgen_key_of(km, n_s, (int64_t)(ddqgen_hash(seed, TH_LINEITEM, DRH_SUPP, (uint64_t)i) % (uint64_t)n_s));
            break;
          case L_LINENUMBER: o32[k] = (int32_t)(i % 4 + 1); break;
          case L_QUANTITY: o64[k] = qty; break;
          case L_EXTENDEDPRICE: o64[k] = (qty / 100) * retailprice_h(pk); break;
          case L_DISCOUNT: o64[k] = (int64_t)(ddqgen_hash(seed, TH_LINEITEM, DRH_DISC, (uint64_t)i) % 11u); break;
          case L_TAX: o64[k] = (int64_t)(ddqgen_hash(seed, TH_LINEITEM, DRH_TAX, (uint64_t)i) % 9u); break;
          case L_RETURNFLAG: /* dict "A","N","R" */
            if (ddqgen_datekey_of_index(rcpt) <= CUTOFF_19950617)
              o32[k] = (ddqgen_hash(seed, TH_LINEITEM, DRH_RFLAG, (uint64_t)i) & 1u) ? 2 : 0;
            else o32[k] = 1;
            break;
          case L_LINESTATUS: /* dict "F","O" */
            o32[k] = ddqgen_datekey_of_index(ship) > CUTOFF_19950617 ? 1 : 0; break;
          case L_SHIPDATE: o32[k] = ddqgen_datekey_of_index(ship); break;
          case L_COMMITDATE:
            o32[k] = ddqgen_datekey_of_index(od + 30 + (int64_t)(ddqgen_hash(seed, TH_LINEITEM, DRH_COMMIT, (uint64_t)i) % 61u));
            break;
          case L_RECEIPTDATE: o32[k] = ddqgen_datekey_of_index(rcpt); break;
        }
      } break;
    }
  }
}

int ddqgen_tpch_column_k(uint64_t seed, double sf, int table, int col, int64_t row_begin,
                         int64_t row_end, void* out, int nthreads, int key_mode) {
  (void)ddqgen_dict_size(0); /* make sure dictionaries are initialised */
  int w = ddqgen_tpch_width(table, col);
  int64_t n = ddqgen_tpch_rows(table, sf);
  if (w == 0 || row_begin < 0 || row_end > n || row_begin > row_end) return -1;
  int64_t total = row_end - row_begin;
  const int64_t chunk = 1 << 16;
  int64_t nchunks = (total + chunk - 1) / chunk, c;
  if (nthreads <= 0) nthreads = 1;
#pragma omp parallel for schedule(dynamic, 4) num_threads(nthreads)
  for (c = 0; c < nchunks; c++) {
    int64_t b = row_begin + c * chunk, e = b + chunk < row_end ? b + chunk : row_end;
    gen_rows_h(seed, sf, table, col, b, e, (char*)out + (b - row_begin) * w, key_mode);
  }
  return 0;
}
int ddqgen_tpch_column(uint64_t seed, double sf, int table, int col, int64_t row_begin,
                       int64_t row_end, void* out, int nthreads) {
  return ddqgen_tpch_column_k(seed, sf, table, col, row_begin, row_end, out, nthreads, 0);
}
